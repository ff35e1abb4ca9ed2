"""Parity of the library's model (mp_predict / mp_select, host C++ behind the C ABI)
with the CPU oracle (oracle/model.py) on seeded synthetic parameter tables.

Bar (BASELINE.json north star + DESIGN.md C17): predictions within 1e-9 relative in
fp64; selected shares equal up to ±A bytes per path with Σ = n exactly; chunk counts
equal; the linearised level within 1e-9.  Host-only, runs without a GPU."""
import math
import random

import pytest

import synth
from oracle import model as M
from paper_conf_sc_sojoodiasfga25_b200 import mp

MiB = 1 << 20
MODES = [M.PAPER, M.B200]


def rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


def setup_pair(ctx, tbl, port):
    paths = [(t["kind"], t["via"]) for t in tbl]
    params = [{k: t[k] for k in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")} for t in tbl]
    for p in params:
        if math.isinf(p["beta2"]):
            p["beta2"] = 0.0          # unused for the direct path
    ctx.set_model(0, 1, paths, params, port)


def oracle_paths(tbl):
    return [M.Path(**t) for t in tbl]


def opts_for(mode, stagger, refine, slot=64 * MiB):
    return M.Options(mode=mode, stagger=bool(stagger), refine=refine, slot_bytes=slot)


CASES = [(seed, nrel, host, mode, stagger, refine)
         for seed in range(6) for nrel in (1, 2, 6) for host in (True, False)
         for mode in MODES for stagger in (0, 1) for refine in (None, False, True)
         if (seed + nrel + stagger) % 2 == 0]


@pytest.mark.parametrize("seed,nrel,host,mode,stagger,refine", CASES)
def test_select_and_predict_parity(seed, nrel, host, mode, stagger, refine):
    tbl = synth.topology(1000 + seed, nrel, host)
    port = dict(alpha=1.5e-6, beta=850e9)
    paths = oracle_paths(tbl)
    oport = M.Port(**port)
    o = opts_for(mode, stagger, refine)
    with mp.Context(world=8, rank=0, model_only=True) as c:
        # the C side resolves (0,1) to direct + 6 relays + host; install our table
        setup_pair(c, tbl, port)
        c.set_options(mode=mode, stagger=stagger, refine=-1 if refine is None else int(refine),
                      slot_bytes=o.slot_bytes)
        rng = random.Random(seed)
        for n in (1, 4096, MiB + 17, 16 * MiB, 64 * MiB + 3, 1 << 30, (2 << 30) - 1):
            cfg = c.select(0, 1, n)
            d = cfg.as_dict()
            ref = M.select(n, paths, o, oport)
            assert sum(d["bytes"]) == n
            for a, b in zip(d["bytes"], ref.bytes):
                assert abs(a - b) <= o.align
            assert rel(d["t_level"], ref.t_level) < 1e-9
            if d["bytes"] == ref.bytes:
                assert d["chunks"] == ref.chunks
                assert rel(d["t_pred"], ref.t_pred) < 1e-9
            # prediction parity on the library's own config and on random configs
            t_o = M.evaluate(n, d["bytes"], d["chunks"], paths, o, oport)
            assert rel(d["t_pred"], t_o) < 1e-9
            for _ in range(3):
                w = [rng.random() for _ in paths]
                nb = [int(n * x / sum(w)) for x in w]
                nb[0] += n - sum(nb)
                ks = [1] + [rng.randint(1, 64) for _ in paths[1:]]
                ccfg = c.make_config(nb, ks, 0, 1)
                assert rel(c.predict(0, 1, n, ccfg), M.evaluate(n, nb, ks, paths, o, oport)) < 1e-9


@pytest.mark.parametrize("mask", [0b1, 0b11, 0b101, 0b1001, 0b1111])
def test_mask_parity(mask):
    tbl = synth.topology(77, 2, True)
    paths = oracle_paths(tbl)
    with mp.Context(world=4, rank=0, model_only=True) as c:
        setup_pair(c, tbl, None)
        n = 256 * MiB
        d = c.select(0, 1, n, mask).as_dict()
        ref = M.select(n, paths, M.Options(), None, [bool(mask >> i & 1) for i in range(4)])
        for a, b in zip(d["bytes"], ref.bytes):
            assert abs(a - b) <= 256
        for i in range(1, 4):
            if not (mask >> i & 1):
                assert d["bytes"][i] == 0


def test_golden_cases_through_the_abi():
    # G2 (Eq 8) and G3 (Eq 11) through mp_select / mp_predict
    us, gbs = 1e-6, 1e9
    with mp.Context(world=3, rank=0, model_only=True) as c:
        c.set_options(stagger=0, align=1, c_min=0, refine=0)
        # G3: direct (1 µs, 100 GB/s) + staged (1, 100, ε 2, α' 1, β' 100), n = 3e6 -> 22 µs.
        # k = 1 reproduces the unpipelined Eq 2 (Eq 13 with k = 1 is Eq 2).
        c.set_model(0, 1, [(0, -1), (1, 2)],
                    [dict(alpha=1 * us, beta=100 * gbs),
                     dict(alpha=1 * us, beta=100 * gbs, alpha2=1 * us, beta2=100 * gbs, eps=2 * us)])
        cfg = c.make_config([2_100_000, 900_000], [1, 1], 0, 1)
        assert rel(c.predict(0, 1, 3_000_000, cfg), 22 * us) < 1e-12
        # G1 (Eq 1): a single direct path
        c.set_model(0, 1, [(0, -1)], [dict(alpha=2 * us, beta=50 * gbs)])
        d = c.select(0, 1, 1_000_000).as_dict()
        assert d["bytes"] == [1_000_000] and rel(d["t_pred"], 22 * us) < 1e-12


def test_cache_invalidation():
    tbl = synth.topology(5, 2, True)
    with mp.Context(world=4, rank=0, model_only=True) as c:
        setup_pair(c, tbl, None)
        a = c.select(0, 1, 64 * MiB).as_dict()
        assert c.select(0, 1, 64 * MiB).as_dict() == a       # cached (C10)
        tbl[0]["beta"] *= 2
        setup_pair(c, tbl, None)
        b = c.select(0, 1, 64 * MiB).as_dict()
        assert b["bytes"][0] > a["bytes"][0]


def test_env_path_filter(monkeypatch):
    # environment variables include / exclude paths (MPX_PATHS, read at mp_init)
    tbl = synth.topology(11, 2, True)
    monkeypatch.setenv("MPX_PATHS", "direct,host")
    with mp.Context(world=4, rank=0, model_only=True) as c:
        setup_pair(c, tbl, None)
        d = c.select(0, 1, 512 * MiB).as_dict()
        assert d["bytes"][1] == 0 and d["bytes"][2] == 0 and d["bytes"][3] > 0
        ref = M.select(512 * MiB, oracle_paths(tbl), M.Options(), None, [True, False, False, True])
        for a, b in zip(d["bytes"], ref.bytes):
            assert abs(a - b) <= 256
    monkeypatch.setenv("MPX_PATHS", "all")
    with mp.Context(world=4, rank=0, model_only=True) as c:
        setup_pair(c, tbl, None)
        assert all(b > 0 for b in c.select(0, 1, 512 * MiB).as_dict()["bytes"])


@pytest.mark.parametrize("seed", range(24))
def test_b200_heavy_latency_parity(seed):
    # reading C26 on the heavy-latency corner (the bottleneck stage flips with the
    # chunk size): library = oracle — shares ±A, chunks, level and prediction 1e-9
    import sys
    import os
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_oracle_select import heavy_paths
    rnd = random.Random(5000 + seed)
    paths = heavy_paths(rnd, 1 + seed % 3)
    tbl = [dict(kind=p.kind, via=(p.via if p.kind == 1 else -1), alpha=p.alpha, beta=p.beta, alpha2=p.alpha2,
                beta2=p.beta2, eps=p.eps, c=p.c, sigma=p.sigma, w=p.w) for p in paths]
    port = dict(alpha=paths[0].alpha, beta=paths[0].beta * rnd.uniform(0.9, 1.1))
    o = M.Options(mode=M.B200, slot_bytes=32 * MiB - 512)
    with mp.Context(world=8, rank=0, model_only=True) as c:
        setup_pair(c, tbl, port)
        c.set_options(mode=M.B200, slot_bytes=o.slot_bytes)
        for n in (16 * MiB, 64 * MiB + 3, 256 * MiB, 1 << 30):
            d = c.select(0, 1, n).as_dict()
            ref = M.select(n, paths, o, M.Port(**port))
            assert sum(d["bytes"]) == n
            for a, b in zip(d["bytes"], ref.bytes):
                assert abs(a - b) <= o.align
            if d["bytes"] == ref.bytes:
                assert d["chunks"] == ref.chunks
            assert rel(d["t_pred"], ref.t_pred) < 1e-9 and rel(d["t_level"], ref.t_level) < 1e-9


@pytest.mark.parametrize("seed", range(24))
def test_c28_wake_parity(seed):
    # reading C28 (a relay that starts A after the message): library = oracle for the
    # pick (shares ±A, chunks, level, prediction 1e-9) and for mp_predict of any config
    import sys
    import os
    import dataclasses
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_oracle_select import heavy_paths, with_wake
    rnd = random.Random(6000 + seed)
    base = heavy_paths(rnd, 1 + seed % 3) if seed % 2 else [M.Path(**t) for t in synth.topology(seed, 3, True)]
    paths = [with_wake(p, rnd) for p in base]
    tbl = [dict(kind=p.kind, via=(p.via if p.kind == 1 else -1), alpha=p.alpha, beta=p.beta, alpha2=p.alpha2,
                beta2=p.beta2, eps=p.eps, c=p.c, sigma=p.sigma, w=p.w) for p in paths]
    port = dict(alpha=paths[0].alpha, beta=paths[0].beta * rnd.uniform(0.9, 1.6))
    o = M.Options(mode=M.B200, slot_bytes=32 * MiB - 512)
    with mp.Context(world=8, rank=0, model_only=True) as c:
        params = [{k: t[k] for k in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")} for t in tbl]
        for p, q in zip(params, paths):
            p["wake"] = q.wake
            if math.isinf(p["beta2"]):
                p["beta2"] = 0.0
        c.set_model(0, 1, [(t["kind"], t["via"]) for t in tbl], params, port)
        assert [p["wake"] for p in c.get_model(0, 1)[1]] == [q.wake for q in paths]
        c.set_options(mode=M.B200, slot_bytes=o.slot_bytes)
        for n in (4 * MiB, 16 * MiB, 64 * MiB + 3, 256 * MiB, 1 << 30):
            d = c.select(0, 1, n).as_dict()
            ref = M.select(n, paths, o, M.Port(**port))
            assert sum(d["bytes"]) == n
            for a, b in zip(d["bytes"], ref.bytes):
                assert abs(a - b) <= o.align
            if d["bytes"] == ref.bytes:
                assert d["chunks"] == ref.chunks
            assert rel(d["t_pred"], ref.t_pred) < 1e-9 and rel(d["t_level"], ref.t_level) < 1e-9
            # mp_predict of an arbitrary config: every staged path at k = 1..8 chunks
            nb = [n - sum(n // (2 * len(paths)) // 256 * 256 for _ in paths[1:])] + \
                 [n // (2 * len(paths)) // 256 * 256] * (len(paths) - 1)
            ch = [1] + [1 + rnd.randrange(8)] * (len(paths) - 1)
            cfg = c.make_config(nb, ch, 0, 1)
            assert rel(c.predict(0, 1, n, cfg), M.evaluate(n, nb, ch, paths, o, M.Port(**port))) < 1e-9
        # wake = 0 is C26 exactly
        c.set_model(0, 1, [(t["kind"], t["via"]) for t in tbl], [dict(p, wake=0.0) for p in params], port)
        d = c.select(0, 1, 256 * MiB).as_dict()
        ref = M.select(256 * MiB, [dataclasses.replace(p, wake=0.0) for p in paths], o, M.Port(**port))
        assert rel(d["t_pred"], ref.t_pred) < 1e-9


def test_c28_wake_validation_and_params_file(tmp_path):
    tbl = synth.topology(3, 2, True)
    paths = [(t["kind"], t["via"]) for t in tbl]
    params = [{k: (0.0 if k == "beta2" and math.isinf(t[k]) else t[k])
               for k in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")} for t in tbl]
    params[1]["wake"] = 17e-6
    f = str(tmp_path / "p.txt")
    with mp.Context(world=4, rank=0, model_only=True) as c:
        for bad in (-1e-6, math.inf, math.nan):
            with pytest.raises(mp.MPError):
                c.set_model(0, 1, paths, [dict(p, wake=bad) if i == 1 else p for i, p in enumerate(params)])
        c.set_model(0, 1, paths, params)
        c.save_params(f)
    with mp.Context(world=4, rank=0, model_only=True) as c:
        c.load_params(f)
        assert c.get_model(0, 1)[1][1]["wake"] == 17e-6
    # a round-2 file (11 fields per path line) still loads, with wake = 0
    txt = open(f).read().splitlines()
    old = [" ".join(ln.split()[:11]) if ln.startswith("path ") else ln for ln in txt]
    open(f, "w").write("\n".join(old) + "\n")
    with mp.Context(world=4, rank=0, model_only=True) as c:
        c.load_params(f)
        assert c.get_model(0, 1)[1][1]["wake"] == 0.0
