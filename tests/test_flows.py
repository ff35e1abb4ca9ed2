"""NEXT f1 — concurrent flows (reading C19, MaxRate-style fair share): pins of the
oracle (oracle/flows.py) and parity of mp_select_flows with it.  CPU only."""
import math
import random

import pytest

import synth
from oracle import flows as OF
from oracle import model as M
from paper_conf_sc_sojoodiasfga25_b200 import mp

MiB = 1 << 20
W = 8


def table(s, d, seed=0):
    """Per-pair parameter table in A1 order: direct, relays (ranks ∉ {s, d}), host."""
    relays = [r for r in range(W) if r not in (s, d)]
    tbl = synth.topology(seed + 100 * s + d, len(relays), True)
    for t, r in zip(tbl[1:1 + len(relays)], relays):
        t["via"] = r
    return tbl


def oracle_env(seed=0, port_beta=850e9):
    def paths(s, d):
        return [M.Path(**t) for t in table(s, d, seed)]

    def port(s, d):
        return M.Port(alpha=1e-6, beta=port_beta)
    return paths, port


def rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


def test_single_flow_is_plain_selection():
    paths, port = oracle_env(1)
    opts = M.Options(mode=M.B200)
    f = OF.select_flows([(0, 1, 256 * MiB, [True] * W)], paths, port, opts)[0]
    ref = M.select(256 * MiB, paths(0, 1), opts, port(0, 1))
    assert f.bytes == ref.bytes and f.t_pred == ref.t_pred


def test_fan_out_divides_the_source_egress():
    # k flows out of GPU 0, direct path only: each gets β/k — T = α + n k / β (Eq 1)
    paths, port = oracle_env(2)
    k, n = 4, 128 * MiB
    flows = [(0, d, n, [True] + [False] * (W - 1)) for d in range(1, k + 1)]
    out = OF.select_flows(flows, paths, port, M.Options(mode=M.PAPER, stagger=False))
    for (s, d, _, _), cfg in zip(flows, out):
        p = paths(s, d)[0]
        assert cfg.bytes[0] == n
        assert rel(cfg.t_pred, p.alpha + n * k / p.beta) < 1e-12


def test_all_gpus_busy_excludes_every_relay():
    # config 5's primary reading: disjoint pairs exchanging both ways cover every GPU
    paths, port = oracle_env(3)
    flows = [(s, s ^ 1, 256 * MiB, [True] * W) for s in range(W)]
    for cfg in OF.select_flows(flows, paths, port, M.Options(mode=M.PAPER)):
        assert all(b == 0 for b in cfg.bytes[1:W - 1])     # relays excluded
        assert cfg.bytes[-1] > 0                           # the PCIe host path survives


def test_idle_gpus_remain_relays():
    paths, port = oracle_env(4)
    out = OF.select_flows([(0, 1, 512 * MiB, [True] * W), (2, 3, 512 * MiB, [True] * W)], paths, port,
                          M.Options(mode=M.PAPER))
    for cfg in out:
        assert any(b > 0 for b in cfg.bytes[1:W - 1])


def random_flows(rng, nf):
    flows = []
    for _ in range(nf):
        s = rng.randrange(W)
        d = rng.choice([x for x in range(W) if x != s])
        mask = [True] + [rng.random() < 0.8 for _ in range(W - 1)]
        flows.append((s, d, rng.choice([64, 256, 1024]) * MiB, mask))
    return flows


@pytest.mark.parametrize("seed", range(10))
def test_fair_share_never_oversubscribes_and_respects_the_lp_bound(seed):
    # B200 mode: at their predicted rates, the selected configs never put more than a
    # link's bandwidth through it (the fair share is feasible jointly), hence the
    # makespan is never below the joint-LP lower bound.
    rng = random.Random(seed)
    B_nvl, B_pcie = 900e9, 60e9
    paths, port = oracle_env(seed, port_beta=B_nvl)
    flows = random_flows(rng, rng.randint(2, 8))
    out = OF.select_flows(flows, paths, port, M.Options(mode=M.B200))
    load = {}
    for (s, d, n, _), cfg in zip(flows, out):
        for i, (p, b) in enumerate(zip(paths(s, d), cfg.bytes)):
            if b == 0:
                continue
            rate = b / cfg.t_pred
            use = {M.DIRECT: [("E", s), ("I", d)],
                   M.GPU_STAGED: [("E", s), ("I", p.via), ("E", p.via), ("I", d)],
                   M.HOST_STAGED: [("U", s), ("D", d)]}[p.kind]
            for u in use:
                load[u] = load.get(u, 0.0) + rate
    for (kind, _), r in load.items():
        assert r <= (B_pcie if kind in "UD" else B_nvl) * (1 + 1e-9), (kind, r)
    lb = OF.lp_lower_bound(flows, paths, B_nvl, B_pcie)
    assert max(c.t_pred for c in out) >= lb * (1 - 1e-9)


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("mode", [M.PAPER, M.B200])
def test_library_parity(seed, mode):
    rng = random.Random(100 + seed)
    flows = random_flows(rng, rng.randint(1, 10))
    paths, port = oracle_env(seed)
    opts = M.Options(mode=mode, slot_bytes=64 * MiB)
    ref = OF.select_flows(flows, paths, port, opts)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=mode, slot_bytes=64 * MiB)
        for s, d in {(s, d) for s, d, _, _ in flows}:
            tbl = table(s, d, seed)
            params = [{k: (0.0 if k == "beta2" and math.isinf(t[k]) else t[k])
                       for k in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")} for t in tbl]
            c.set_model(s, d, [(t["kind"], t["via"]) for t in tbl], params, dict(alpha=1e-6, beta=850e9))
        got = c.select_flows([(s, d, n, sum(1 << i for i, m in enumerate(mask) if m)) for s, d, n, mask in flows])
        for g, r in zip(got, ref):
            gd = g.as_dict()
            assert sum(gd["bytes"]) == sum(r.bytes)
            for a, b in zip(gd["bytes"], r.bytes):
                assert abs(a - b) <= 256
            assert rel(gd["t_level"], r.t_level) < 1e-9
            if gd["bytes"] == r.bytes:
                assert gd["chunks"] == r.chunks and rel(gd["t_pred"], r.t_pred) < 1e-9
