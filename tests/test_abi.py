"""The C-ABI library loads on a CPU-only box and exports every symbol include/mp.h
declares; host-side argument validation works without a GPU."""
import os
import re

import pytest

from paper_conf_sc_sojoodiasfga25_b200 import mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "mp.h")).read()
    return sorted(set(re.findall(r"^\s*(?:int|const char \*)\s*(mp_\w+)\s*\(", src, re.M)))


def test_header_symbols_exported():
    L = mp.lib()
    names = declared_symbols()
    assert len(names) >= 20
    for n in names:
        assert hasattr(L, n), n
    assert sorted(mp.exported_symbols()) == names
    assert L.mp_abi_version() == 5


def test_strerror():
    L = mp.lib()
    assert L.mp_strerror(0) == b"MP_OK"
    assert L.mp_strerror(-7) == b"MP_ERR_TIMEOUT"


def test_model_only_context_rejects_engine_calls():
    with mp.Context(model_only=True) as c:
        with pytest.raises(mp.MPError) as e:
            c.alloc(1024)
        assert e.value.status == -5
        with pytest.raises(mp.MPError):
            c.xfer(0, 0, 16)
        with pytest.raises(mp.MPError) as e:
            c.register(0x1000, 4096)
        assert e.value.status == -5
        with pytest.raises(mp.MPError):
            c.deregister(1)


def test_init_validation():
    with pytest.raises(mp.MPError):
        mp.Context(rank=2, world=2, model_only=True)


def test_paths_order_A1():
    with mp.Context(world=8, rank=0, model_only=True) as c:
        ps = c.paths(0, 1)
        assert ps[0] == (mp.MP_PATH_DIRECT, -1)
        assert ps[1:7] == [(mp.MP_PATH_GPU, r) for r in range(2, 8)]
        assert ps[7] == (mp.MP_PATH_HOST, -1)
    with mp.Context(world=1, model_only=True, n_loop_relays=2, host_path=0) as c:
        assert c.paths(0, 0) == [(0, -1), (1, 0), (1, 1)]


def test_set_model_validation():
    with mp.Context(world=2, rank=0, model_only=True) as c:
        ok = dict(alpha=1e-6, beta=1e11)
        with pytest.raises(mp.MPError):
            c.set_model(0, 1, [(mp.MP_PATH_GPU, 0)], [ok])        # paths[0] must be direct
        with pytest.raises(mp.MPError):
            c.set_model(0, 1, [(0, -1)], [dict(alpha=1e-6, beta=0)])
        with pytest.raises(mp.MPError):                            # staged needs ε + α' > 0
            c.set_model(0, 1, [(0, -1), (2, -1)], [ok, dict(alpha=1e-6, beta=1e10, beta2=1e10)])
        c.set_model(0, 1, [(0, -1)], [ok])
        cfg = c.make_config([1000], [1], 0, 1)
        with pytest.raises(mp.MPError):
            c.predict(0, 1, 999, cfg)                              # Σ bytes != n
        assert abs(c.predict(0, 1, 1000, cfg) - (1e-6 + 1000 / 1e11)) < 1e-18


def test_params_roundtrip(tmp_path):
    with mp.Context(world=3, rank=0, model_only=True) as c:
        ps = c.paths(0, 1)
        prm = [dict(alpha=1.5e-6, beta=7e11, w=1)] + [dict(alpha=2e-6, beta=6e11, alpha2=1e-6, beta2=5e11,
                                                           eps=3e-6, w=1)] + [dict(alpha=5e-6, beta=5e10,
                                                                                   alpha2=4e-6, beta2=4e10,
                                                                                   eps=2e-6)]
        c.set_model(0, 1, ps, prm, dict(alpha=1e-6, beta=9e11))
        f = str(tmp_path / "p.txt")
        c.save_params(f)
        with mp.Context(world=3, rank=0, model_only=True) as d:
            d.load_params(f)
            assert d.get_model(0, 1) == c.get_model(0, 1)
