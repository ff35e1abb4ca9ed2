"""NEXT f2 — parity of the library's window model (mp_predict_window, mp_select_window,
reading C24) and host duplex factor (mp_set_host_duplex in mp_select_flows, reading
C25) with the oracle (oracle/window.py).  CPU only (model-only contexts)."""
import math
import os
import random

import pytest

import synth
from oracle import model as M
from oracle import window as WN
from paper_conf_sc_sojoodiasfga25_b200 import mp

MiB = 1 << 20
W = 4
FIELDS = ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")


def rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


def table(s, d, seed=0):
    relays = [r for r in range(W) if r not in (s, d)]
    tbl = synth.topology(seed + 10 * s + d, len(relays), True)
    for t, r in zip(tbl[1:1 + len(relays)], relays):
        t["via"] = r
    return tbl


def install(c, s, d, tbl, port):
    params = [{k: (0.0 if k == "beta2" and math.isinf(t[k]) else t[k]) for k in FIELDS} for t in tbl]
    c.set_model(s, d, [(t["kind"], t["via"]) for t in tbl], params,
                None if port is None else dict(alpha=port.alpha, beta=port.beta))


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("mode", [M.PAPER, M.B200])
def test_select_and_predict_window_parity(seed, mode):
    rng = random.Random(seed)
    tbl = table(0, 1, seed)
    paths = [M.Path(**t) for t in tbl]
    port = M.Port(alpha=rng.uniform(1, 4) * 1e-6, beta=850e9)
    h = [rng.uniform(0, 1.5) * p.alpha for p in paths]
    tau = rng.uniform(0, 10e-6)
    opts = M.Options(mode=mode, slot_bytes=64 * MiB)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=mode, slot_bytes=64 * MiB)
        install(c, 0, 1, tbl, port)
        c.set_window_model(0, 1, h, tau)
        hh, tt = c.get_window_model(0, 1)
        assert hh == h and tt == tau
        for n in (1 * MiB + 17, 16 * MiB, 64 * MiB, 1024 * MiB):
            for w in (1, 2, 16, 64):
                ref = WN.select_window(n, w, paths, h, opts, port, tau=tau)
                got = c.select_window(0, 1, n, w).as_dict()
                assert sum(got["bytes"]) == n
                for a, b in zip(got["bytes"], ref.bytes):
                    assert abs(a - b) <= 256
                assert rel(got["t_level"], ref.t_level) < 1e-9
                if got["bytes"] == ref.bytes:
                    assert got["chunks"] == ref.chunks and rel(got["t_pred"], ref.t_pred) < 1e-9
                # mp_predict_window on the oracle's config
                cfg = c.make_config(ref.bytes, ref.chunks, 0, 1)
                t = c.predict_window(0, 1, n, w, cfg)
                assert rel(t, WN.evaluate_window(n, w, ref.bytes, ref.chunks, paths, h, opts, port, tau)) < 1e-9
                if w == 1:
                    assert rel(t, c.predict(0, 1, n, cfg) + tau) < 1e-12


def test_window_option_makes_mp_select_window_aware():
    tbl = table(0, 1, 3)
    paths = [M.Path(**t) for t in tbl]
    h = [0.8 * p.alpha for p in paths]
    with mp.Context(world=W, rank=0, model_only=True) as c:
        install(c, 0, 1, tbl, M.Port(alpha=2e-6, beta=850e9))
        c.set_window_model(0, 1, h, 1e-6)
        n = 8 * MiB
        per_msg = c.select(0, 1, n).as_dict()
        c.set_options(window=16)
        assert c.get_options()["window"] == 16
        got = c.select(0, 1, n).as_dict()
        want = c.select_window(0, 1, n, 16).as_dict()
        assert got == want
        ref = WN.select_window(n, 16, paths, h, M.Options(), M.Port(alpha=2e-6, beta=850e9), tau=1e-6)
        for a, b in zip(got["bytes"], ref.bytes):
            assert abs(a - b) <= 256
        c.set_window_model(0, 1, [0.0] * len(h), 0.0)   # invalidates the cache
        assert c.select(0, 1, n).as_dict()["bytes"] == per_msg["bytes"]
        c.set_options(window=1)
        assert c.select(0, 1, n).as_dict() == per_msg


def test_window_defaults_and_errors():
    with mp.Context(world=W, rank=0, model_only=True) as c:
        n = 64 * MiB
        base = c.select(0, 1, n).as_dict()
        for w in (1, 8):  # no window model installed: h = 0, τ = 0 → w × the message
            got = c.select_window(0, 1, n, w).as_dict()
            assert got["bytes"] == base["bytes"] and rel(got["t_pred"], w * base["t_pred"]) < 1e-12
        h, tau = c.get_window_model(0, 1)
        assert h == [0.0] * len(c.paths(0, 1)) and tau == 0.0
        with pytest.raises(mp.MPError):
            c.select_window(0, 1, n, 0)
        with pytest.raises(mp.MPError):
            c.set_window_model(0, 1, [1e-6], 0.0)           # wrong path count
        with pytest.raises(mp.MPError):
            c.set_window_model(0, 1, [-1.0] * len(h), 0.0)  # h < 0
        with pytest.raises(mp.MPError):
            c.set_host_duplex(0, 0.0)
        with pytest.raises(mp.MPError):
            c.set_host_duplex(0, 1.5)
        assert c.get_host_duplex(3) == 1.0


def test_window_and_duplex_survive_the_params_file(tmp_path):
    f = str(tmp_path / "p.txt")
    with mp.Context(world=W, rank=0, model_only=True) as c:
        h = [float(i + 1) * 1e-6 for i in range(len(c.paths(0, 1)))]
        c.set_window_model(0, 1, h, 3e-6)
        c.set_host_duplex(2, 0.75)
        c.save_params(f)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.load_params(f)
        assert c.get_window_model(0, 1) == (h, 3e-6)
        assert c.get_host_duplex(2) == 0.75 and c.get_host_duplex(1) == 1.0


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("mode", [M.PAPER, M.B200])
def test_select_flows_duplex_parity(seed, mode):
    rng = random.Random(50 + seed)
    kappa = {g: rng.choice([1.0, rng.uniform(0.5, 1.0)]) for g in range(W)}
    flows = []
    for _ in range(rng.randint(1, 6)):
        s = rng.randrange(W)
        d = rng.choice([x for x in range(W) if x != s])
        mask = [True] + [rng.random() < 0.8 for _ in range(W - 1)]
        flows.append((s, d, rng.choice([16, 64, 256]) * MiB, mask))
    if rng.random() < 0.5:  # a bidirectional pair
        flows.append((flows[0][1], flows[0][0], flows[0][2], flows[0][3]))

    def paths(s, d):
        return [M.Path(**t) for t in table(s, d, seed)]

    def port(s, d):
        return M.Port(alpha=1e-6, beta=850e9)
    opts = M.Options(mode=mode, slot_bytes=64 * MiB)
    ref = WN.select_flows_duplex(flows, paths, port, opts, kappa.get)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=mode, slot_bytes=64 * MiB)
        for g, k in kappa.items():
            c.set_host_duplex(g, k)
        for s, d in {(s, d) for s, d, _, _ in flows}:
            install(c, s, d, table(s, d, seed), port(s, d))
        got = c.select_flows([(s, d, n, sum(1 << i for i, m in enumerate(mask) if m)) for s, d, n, mask in flows])
        for g, r in zip(got, ref):
            gd = g.as_dict()
            assert sum(gd["bytes"]) == sum(r.bytes)
            for a, b in zip(gd["bytes"], r.bytes):
                assert abs(a - b) <= 256
            assert rel(gd["t_level"], r.t_level) < 1e-9
            if gd["bytes"] == r.bytes:
                assert gd["chunks"] == r.chunks and rel(gd["t_pred"], r.t_pred) < 1e-9


@pytest.mark.parametrize("mode", [M.PAPER, M.B200])
def test_window_model_applies_to_every_size_band(mode):
    # C24 with C20: the pair's h and τ hold for every band; a_i = min(h_i, α_i) takes
    # the α of n's band (oracle: oracle/bands.band_index + oracle/window.select_window).
    from oracle import bands as OB
    rng = random.Random(7)
    base = [M.Path(**t) for t in table(0, 1, 11)]
    scaled = [M.Path(**{**t, "alpha": t["alpha"] * 0.3, "alpha2": t["alpha2"] * 0.3}) for t in table(0, 1, 11)]
    bands = [(0, scaled, M.Port(1e-6, 8e11)), (16 * MiB, base, M.Port(3e-6, 9e11))]
    h = [rng.uniform(0.2, 1.2) * p.alpha for p in base]
    tau = 2e-6
    opts = M.Options(mode=mode, slot_bytes=64 * MiB)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=mode, slot_bytes=64 * MiB)
        install(c, 0, 1, table(0, 1, 11), None)
        prm = [{k: (0.0 if k == "beta2" and math.isinf(getattr(p, k)) else getattr(p, k)) for k in FIELDS}
               for p in scaled]
        c.set_model(0, 1, [(p.kind, p.via) for p in scaled], prm, dict(alpha=1e-6, beta=8e11))
        prm = [{k: (0.0 if k == "beta2" and math.isinf(getattr(p, k)) else getattr(p, k)) for k in FIELDS}
               for p in base]
        c.set_model_band(0, 1, 16 * MiB, prm, dict(alpha=3e-6, beta=9e11))
        c.set_window_model(0, 1, h, tau)
        for n in (4 * MiB, 16 * MiB - 256, 16 * MiB, 256 * MiB):
            j = OB.band_index([b[0] for b in bands], n)
            _, ps, port = bands[j]
            for w in (1, 8):
                ref = WN.select_window(n, w, ps, h, opts, port, tau=tau)
                got = c.select_window(0, 1, n, w).as_dict()
                for a, b in zip(got["bytes"], ref.bytes):
                    assert abs(a - b) <= 256
                assert rel(got["t_level"], ref.t_level) < 1e-9
                if got["bytes"] == ref.bytes:
                    assert rel(got["t_pred"], ref.t_pred) < 1e-9


def test_predict_window_rejects_bad_configs():
    with mp.Context(world=W, rank=0, model_only=True) as c:
        n = 8 * MiB
        ps = c.paths(0, 1)
        bad = c.make_config([n - 1] + [0] * (len(ps) - 1), [1] + [0] * (len(ps) - 1), 0, 1)
        with pytest.raises(mp.MPError):
            c.predict_window(0, 1, n, 4, bad)                   # bytes do not sum to n
        ok = c.make_config([n] + [0] * (len(ps) - 1), [1] + [0] * (len(ps) - 1), 0, 1)
        with pytest.raises(mp.MPError):
            c.predict_window(0, 1, n, 0, ok)                    # window 0
        assert c.predict_window(0, 1, n, 4, ok) == pytest.approx(4 * c.predict(0, 1, n, ok), rel=1e-12)


@pytest.mark.parametrize("seed", range(6))
def test_select_flows_with_window_option_parity(seed):
    # mp_model_opts.window > 1 makes mp_select_flows window-aware too (C24 with C19/C25)
    rng = random.Random(300 + seed)
    flows = []
    for _ in range(rng.randint(1, 5)):
        s = rng.randrange(W)
        d = rng.choice([x for x in range(W) if x != s])
        flows.append((s, d, rng.choice([4, 16, 64]) * MiB, [True] * W))
    kappa = {g: rng.uniform(0.6, 1.0) for g in range(W)}
    wins = {}

    def paths(s, d):
        return [M.Path(**t) for t in table(s, d, seed)]

    def port(s, d):
        return M.Port(alpha=1e-6, beta=850e9)

    def window_of(s, d):
        if (s, d) not in wins:
            r = random.Random(1000 * s + d + seed)
            wins[(s, d)] = ([r.uniform(0, 1.2) * p.alpha for p in paths(s, d)], r.uniform(0, 5e-6))
        return wins[(s, d)]
    opts = M.Options(mode=M.B200, slot_bytes=64 * MiB)
    ref = WN.select_flows_duplex(flows, paths, port, opts, kappa.get, window=8, window_of=window_of)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=M.B200, slot_bytes=64 * MiB, window=8)
        for g, k in kappa.items():
            c.set_host_duplex(g, k)
        for s, d in {(s, d) for s, d, _, _ in flows}:
            install(c, s, d, table(s, d, seed), port(s, d))
            h, tau = window_of(s, d)
            c.set_window_model(s, d, h, tau)
        got = c.select_flows([(s, d, n, 0) for s, d, n, _ in flows])
        for g, r in zip(got, ref):
            gd = g.as_dict()
            for a, b in zip(gd["bytes"], r.bytes):
                assert abs(a - b) <= 256
            assert rel(gd["t_level"], r.t_level) < 1e-9
            if gd["bytes"] == r.bytes:
                assert gd["chunks"] == r.chunks and rel(gd["t_pred"], r.t_pred) < 1e-9


def test_params_file_with_bands_window_and_duplex(tmp_path):
    f = str(tmp_path / "p.txt")
    with mp.Context(world=W, rank=0, model_only=True) as c:
        tbl = table(0, 1, 5)
        install(c, 0, 1, tbl, M.Port(alpha=1e-6, beta=8e11))
        prm = [{k: (0.0 if k == "beta2" and math.isinf(t[k]) else t[k] * (0.5 if k == "alpha" else 1.0))
                for k in FIELDS} for t in tbl]
        c.set_model_band(0, 1, 8 * MiB, prm, dict(alpha=2e-6, beta=9e11))
        h = [0.5 * t["alpha"] for t in tbl]
        c.set_window_model(0, 1, h, 1.5e-6)
        c.set_host_duplex(3, 0.6)
        want = [c.select_window(0, 1, n, 16).as_dict() for n in (2 * MiB, 64 * MiB)]
        c.save_params(f)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.load_params(f)
        assert [b[0] for b in c.get_model_bands(0, 1)] == [0, 8 * MiB]
        assert c.get_window_model(0, 1) == (h, 1.5e-6) and c.get_host_duplex(3) == 0.6
        got = [c.select_window(0, 1, n, 16).as_dict() for n in (2 * MiB, 64 * MiB)]
        assert got == want


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("mode", [M.PAPER, M.B200])
def test_submission_time_parity(seed, mode):
    # reading C27: the context's host submission time enters every window prediction
    # (mp_predict_window, mp_select_window's t_pred) as the oracle's h_sub; it survives
    # the parameter file; 0 is C24
    rng = random.Random(100 + seed)
    tbl = table(0, 1, seed)
    paths = [M.Path(**t) for t in tbl]
    port = M.Port(alpha=2e-6, beta=850e9)
    h = [rng.uniform(0, 1.5) * p.alpha for p in paths]
    tau, h_sub = rng.uniform(0, 10e-6), rng.choice([0.0, 1.5e-6, 3e-6, 40e-6])
    opts = M.Options(mode=mode, slot_bytes=64 * MiB)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=mode, slot_bytes=64 * MiB)
        install(c, 0, 1, tbl, port)
        c.set_window_model(0, 1, h, tau)
        c.set_submit_time(h_sub)
        assert c.get_submit_time() == h_sub
        for n in (64 * 1024, 1 * MiB, 16 * MiB):
            for w in (2, 16, 64):
                ref = WN.select_window(n, w, paths, h, opts, port, tau=tau, h_sub=h_sub)
                got = c.select_window(0, 1, n, w).as_dict()
                if got["bytes"] == ref.bytes:
                    assert rel(got["t_pred"], ref.t_pred) < 1e-9
                cfg = c.make_config(ref.bytes, ref.chunks, 0, 1)
                want = WN.evaluate_window(n, w, ref.bytes, ref.chunks, paths, h, opts, port, tau, h_sub)
                assert rel(c.predict_window(0, 1, n, w, cfg), want) < 1e-9
    with pytest.raises(mp.MPError):
        with mp.Context(world=W, rank=0, model_only=True) as c:
            c.set_submit_time(-1.0)


def test_submission_time_survives_the_params_file(tmp_path):
    f = str(tmp_path / "p.txt")
    with mp.Context(world=2, rank=0, model_only=True) as c:
        c.set_submit_time(2.5e-6)
        c.save_params(f)
    with mp.Context(world=2, rank=0, model_only=True) as c:
        c.load_params(f)
        assert c.get_submit_time() == 2.5e-6


@pytest.mark.parametrize("seed", range(8))
def test_c28_window_parity(seed):
    # reading C28 in a window: the relay's start delays the window once (library =
    # oracle for mp_select_window and mp_predict_window); w = 1 is the single message
    import dataclasses
    rng = random.Random(300 + seed)
    tbl = table(0, 1, seed)
    paths = [M.Path(**t) for t in tbl]
    paths = [dataclasses.replace(p, wake=rng.uniform(2e-6, 300e-6)) if p.kind == M.GPU_STAGED else p
             for p in paths]
    port = M.Port(alpha=2e-6, beta=850e9)
    h = [rng.uniform(0, 1.5) * p.alpha for p in paths]
    tau = rng.uniform(0, 10e-6)
    opts = M.Options(mode=M.B200, slot_bytes=64 * MiB)
    with mp.Context(world=W, rank=0, model_only=True) as c:
        c.set_options(mode=M.B200, slot_bytes=64 * MiB)
        params = [{k: (0.0 if k == "beta2" and math.isinf(t[k]) else t[k]) for k in FIELDS} for t in tbl]
        for p, q in zip(params, paths):
            p["wake"] = q.wake
        c.set_model(0, 1, [(t["kind"], t["via"]) for t in tbl], params, dict(alpha=port.alpha, beta=port.beta))
        c.set_window_model(0, 1, h, tau)
        for n in (1 * MiB + 17, 16 * MiB, 64 * MiB, 1024 * MiB):
            for w in (1, 2, 16, 64):
                ref = WN.select_window(n, w, paths, h, opts, port, tau=tau)
                got = c.select_window(0, 1, n, w).as_dict()
                assert sum(got["bytes"]) == n
                for a, b in zip(got["bytes"], ref.bytes):
                    assert abs(a - b) <= 256
                assert rel(got["t_level"], ref.t_level) < 1e-9
                if got["bytes"] == ref.bytes:
                    assert got["chunks"] == ref.chunks and rel(got["t_pred"], ref.t_pred) < 1e-9
                cfg = c.make_config(ref.bytes, ref.chunks, 0, 1)
                t = c.predict_window(0, 1, n, w, cfg)
                assert rel(t, WN.evaluate_window(n, w, ref.bytes, ref.chunks, paths, h, opts, port, tau)) < 1e-9
                if w == 1:
                    assert rel(t, c.predict(0, 1, n, cfg) + tau) < 1e-12
