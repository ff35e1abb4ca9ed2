"""ORACLE (test infrastructure only; see oracle/__init__.py).  NEXT f3: collectives.

PAPER.md §5.3: MPI_Allreduce and MPI_Alltoall run as sequences of
multi-path P2P messages (UCC: K-nomial scatter-reduce + K-nomial allgather for
Allreduce, Bruck for Alltoall).  Whatever the schedule, each reaches a result with a
plain definition (MPI semantics), which is what this module writes out:

  alltoall : recv_r[s·B : (s+1)·B] = send_s[r·B : (r+1)·B]      for every s, r
  allreduce: recv_r = Σ_s send_s   (elementwise, every rank r)

and a plain executor of a *plan* (the library's schedule as data, `mp_coll_plan_build`)
over W simulated ranks with numpy copies — the CPU pin of the schedule logic: a plan
is correct iff executing it literally reproduces the definitions above.
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np


def alltoall(sends: Sequence[np.ndarray], block: int) -> List[np.ndarray]:
    """MPI_Alltoall: rank r receives block r of every rank s, in rank order."""
    W = len(sends)
    return [np.concatenate([sends[s][r * block:(r + 1) * block] for s in range(W)]) if W else
            np.zeros(0, np.uint8) for r in range(W)]


def allreduce_sum(sends: Sequence[np.ndarray]) -> np.ndarray:
    """MPI_Allreduce(MPI_SUM): the elementwise sum over ranks, accumulated in fp64 for
    floating point (int64 for integers) — the exact reference the library's
    reassociated sums are compared with under a rounding bound."""
    acc_t = np.float64 if np.issubdtype(sends[0].dtype, np.floating) else np.int64
    acc = np.zeros(sends[0].shape, dtype=acc_t)
    for s in sends:
        acc += s.astype(acc_t)
    return acc


BUF_SEND, BUF_RECV, BUF_TMP = 0, 1, 2


def execute_plans(plans, sends: Sequence[np.ndarray], recv_bytes: int, dtype=np.uint8):
    """Run per-rank plans in lock step with plain numpy copies: every rank's pre copies,
    then step by step every rank packs its send segments into one message, the message
    goes to `send_to`, whose matching step must name this rank in `recv_from`; it is
    split over the receiver's recv segments (copied, or added elementwise when the step
    reduces); then every rank's post copies.  plans[r] is a dict as returned by
    paper_conf_sc_sojoodiasfga25_b200.mp.coll_plan.  Returns the recv buffers."""
    W = len(plans)
    bufs = []
    for r in range(W):
        bufs.append({BUF_SEND: sends[r].view(np.uint8).copy(),
                     BUF_RECV: np.zeros(recv_bytes, np.uint8),
                     BUF_TMP: np.zeros(plans[r]["tmp_bytes"], np.uint8)})

    def copies(r, lst):
        for c in lst:
            src = bufs[r][c["src_buf"]][c["src_off"]:c["src_off"] + c["len"]].copy()
            bufs[r][c["dst_buf"]][c["dst_off"]:c["dst_off"] + c["len"]] = src

    for r in range(W):
        copies(r, plans[r]["pre"])
    nsteps = plans[0]["nsteps"]
    assert all(p["nsteps"] == nsteps for p in plans), "ranks disagree on the step count"
    for j in range(nsteps):
        msgs = {}
        for r in range(W):
            st = plans[r]["steps"][j]
            if st["send_to"] < 0:
                continue
            parts = [bufs[r][g["buf"]][g["off"]:g["off"] + g["len"]] for g in st["send_segs"]]
            m = np.concatenate(parts) if parts else np.zeros(0, np.uint8)
            assert len(m) == st["bytes"], (r, j)
            msgs[(r, st["send_to"])] = m.copy()
        for r in range(W):
            st = plans[r]["steps"][j]
            if st["recv_from"] < 0:
                continue
            m = msgs.pop((st["recv_from"], r))
            o = 0
            for g in st["recv_segs"]:
                part = m[o:o + g["len"]]
                tgt = bufs[r][g["buf"]][g["off"]:g["off"] + g["len"]]
                if st["reduce"]:
                    tv = tgt.view(dtype)
                    tv += part.view(dtype)
                else:
                    tgt[:] = part
                o += g["len"]
            assert o == len(m), (r, j, o, len(m))
        assert not msgs, f"unmatched messages at step {j}: {list(msgs)}"
    for r in range(W):
        copies(r, plans[r]["post"])
    return [bufs[r][BUF_RECV] for r in range(W)]
