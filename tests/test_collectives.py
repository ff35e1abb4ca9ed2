"""NEXT f3 (§5.3): the collective schedules of the library
(mp_coll_plan_build) executed literally over W simulated ranks by the oracle's plain
plan executor reproduce the MPI definitions (oracle/collectives.py) — Alltoall
bit-exact, Allreduce exact on integers.  CPU only; the GPU executor is tested in
tests/test_world.py (scenario "coll")."""
import numpy as np
import pytest

from oracle import collectives as OCL
from paper_conf_sc_sojoodiasfga25_b200 import mp

ALGOS_A2A = [mp.MP_ALGO_BRUCK, mp.MP_ALGO_PAIRWISE]


def plans(coll, algo, W, nbytes, elem=1):
    return [mp.coll_plan(coll, algo, W, r, nbytes, elem) for r in range(W)]


@pytest.mark.parametrize("W", [1, 2, 3, 4, 5, 6, 7, 8, 9, 12, 16])
@pytest.mark.parametrize("algo", ALGOS_A2A)
@pytest.mark.parametrize("B", [1, 7, 256, 4099])
def test_alltoall_plans_match_definition(W, algo, B):
    rng = np.random.default_rng(1000 * W + B + algo)
    sends = [rng.integers(0, 256, W * B, dtype=np.uint8) for _ in range(W)]
    got = OCL.execute_plans(plans(mp.MP_COLL_ALLTOALL, algo, W, B), sends, W * B)
    exp = OCL.alltoall(sends, B)
    for r in range(W):
        assert np.array_equal(got[r], exp[r]), (W, algo, B, r)


@pytest.mark.parametrize("W", [2, 3, 5, 8, 16])
def test_alltoall_step_counts(W):
    # Bruck: ⌈log2 W⌉ steps (UCC's algorithm); pairwise: W − 1 steps
    assert plans(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_BRUCK, W, 64)[0]["nsteps"] == (W - 1).bit_length()
    assert plans(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_PAIRWISE, W, 64)[0]["nsteps"] == W - 1


@pytest.mark.parametrize("W,algo", [(2, mp.MP_ALGO_KNOMIAL), (4, mp.MP_ALGO_KNOMIAL), (8, mp.MP_ALGO_KNOMIAL),
                                    (16, mp.MP_ALGO_KNOMIAL), (2, mp.MP_ALGO_RING), (3, mp.MP_ALGO_RING),
                                    (5, mp.MP_ALGO_RING), (7, mp.MP_ALGO_RING), (8, mp.MP_ALGO_RING),
                                    (1, mp.MP_ALGO_RING)])
@pytest.mark.parametrize("count", [1, 3, 17, 1000, 4096 + 5])
def test_allreduce_plans_match_definition(W, algo, count):
    rng = np.random.default_rng(W * 7919 + count)
    sends = [rng.integers(-2 ** 31, 2 ** 31, count, dtype=np.int64).astype(np.int32) for _ in range(W)]
    got = OCL.execute_plans(plans(mp.MP_COLL_ALLREDUCE, algo, W, 4 * count, 4), sends, 4 * count, np.int32)
    exp = OCL.allreduce_sum(sends).astype(np.int32)     # int32 wrap-around, as the device
    for r in range(W):
        assert np.array_equal(got[r].view(np.int32), exp), (W, algo, count, r)


@pytest.mark.parametrize("W", [2, 4, 8, 16])
def test_knomial_step_count_and_traffic(W):
    # radix-2 K-nomial: log2 W reduce-scatter + log2 W allgather steps; each rank sends
    # (W−1)/W of the vector in each phase (bandwidth-optimal), the same as the ring
    n = 1 << 16
    p = plans(mp.MP_COLL_ALLREDUCE, mp.MP_ALGO_KNOMIAL, W, 4 * n, 4)[0]
    m = W.bit_length() - 1
    assert p["nsteps"] == 2 * m
    sent = sum(s["bytes"] for s in p["steps"])
    assert sent == 2 * 4 * n * (W - 1) // W
    assert [s["reduce"] for s in p["steps"]] == [1] * m + [0] * m


def test_auto_resolution_and_errors():
    assert mp.coll_plan(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_AUTO, 4, 0, 1024)["algo"] == mp.MP_ALGO_BRUCK
    assert mp.coll_plan(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_AUTO, 4, 0, 1 << 20)["algo"] == mp.MP_ALGO_PAIRWISE
    assert mp.coll_plan(mp.MP_COLL_ALLREDUCE, mp.MP_ALGO_AUTO, 8, 0, 4096, 4)["algo"] == mp.MP_ALGO_KNOMIAL
    assert mp.coll_plan(mp.MP_COLL_ALLREDUCE, mp.MP_ALGO_AUTO, 6, 0, 4096, 4)["algo"] == mp.MP_ALGO_RING
    with pytest.raises(mp.MPError):
        mp.coll_plan(mp.MP_COLL_ALLREDUCE, mp.MP_ALGO_KNOMIAL, 6, 0, 4096, 4)   # W not a power of 2
    with pytest.raises(mp.MPError):
        mp.coll_plan(mp.MP_COLL_ALLREDUCE, mp.MP_ALGO_RING, 4, 0, 4097, 4)      # not whole elements
    with pytest.raises(mp.MPError):
        mp.coll_plan(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_KNOMIAL, 4, 0, 64)
    with pytest.raises(mp.MPError):
        mp.coll_plan(mp.MP_COLL_ALLTOALL, mp.MP_ALGO_BRUCK, 4, 4, 64)           # rank out of range


def test_model_only_context_rejects_collectives():
    with mp.Context(model_only=True) as c:
        with pytest.raises(mp.MPError):
            c.alltoall(0x1000, 0x2000, 64)
        with pytest.raises(mp.MPError):
            c.allreduce(0x1000, 0x2000, 64)
