"""Host-side checks of the emulated world's C ABI (include/mp.h: mp_init_emulated,
mp_emu_run, mp_finalize_emulated) that need no GPU: the flag cannot be set through
mp_init, bad arguments are refused, and a failed bootstrap (no CUDA device here)
returns an error from every rank thread instead of leaving one waiting in the
in-process all-gather."""
import ctypes as C

import pytest

from paper_conf_sc_sojoodiasfga25_b200 import mp


def test_emulated_flag_refused_by_mp_init():
    L = mp.lib()
    a = mp.mp_init_args()
    a.rank, a.world, a.device = 0, 2, 0
    a.flags = mp.MP_INIT_EMULATED | mp.MP_INIT_NO_CALIBRATE
    a.n_loop_relays, a.host_path = -1, -1
    a.allgather = mp.ALLGATHER()
    h = C.c_void_p()
    assert L.mp_init(C.byref(h), C.byref(a)) == mp.MP_ERR_INVALID
    assert not h.value


def test_emulated_bad_arguments():
    L = mp.lib()
    hs = (C.c_void_p * 4)()
    a = mp.mp_init_args()
    a.world = 1  # an emulated world has >= 2 ranks
    a.allgather = mp.ALLGATHER()
    assert L.mp_init_emulated(hs, C.byref(a)) == mp.MP_ERR_INVALID
    a.world, a.flags = 2, mp.MP_INIT_MODEL_ONLY
    assert L.mp_init_emulated(hs, C.byref(a)) == mp.MP_ERR_INVALID
    assert L.mp_emu_run(None, 2, None, None) == mp.MP_ERR_INVALID
    assert L.mp_finalize_emulated(None, 2) == mp.MP_ERR_INVALID


@pytest.mark.timeout(120)
def test_emulated_bootstrap_failure_does_not_hang():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("checks the no-device failure path")
    with pytest.raises(mp.MPError) as e:
        mp.EmulatedWorld(3, heap_bytes=1 << 20, slot_bytes=1 << 20, slots=2, relay_ctas=4)
    assert e.value.status in (mp.MP_ERR_CUDA, mp.MP_ERR_NOMEM, mp.MP_ERR_UNSUPPORTED)
