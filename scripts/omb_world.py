#!/usr/bin/env python3
"""OSU-micro-benchmark-style sweep across GPUs (BASELINE.json config 4: osu_bw /
osu_bibw / osu_latency, 4 KiB - 2 GiB, single pair GPU0 <-> GPU1, vs cudaMemcpyPeer
and NCCL send/recv; the paper's OMB methodology).

    torchrun --nproc-per-node N scripts/omb_world.py [--min-bytes 4096] [--max-bytes 1073741824]
             [--windows 1,16,64] [--out gpurun_out/omb_world.jsonl]

Ranks 0 and 1 are the pair; ranks 2.. serve as relay GPUs for the model's configs.
  bw       a window of w model-selected mp_send calls (mp_recv on the peer), then a
           4-byte ack back (OMB), device time on rank 0's stream; GB/s = n·w / time
  bibw     both directions at once (each rank sends w and receives w on two streams)
  latency  ping-pong, one-way = round trip / 2 (sizes <= 4 MiB)
  ce       the same window as copy-engine peer copies (cudaMemcpyAsync into the
           IPC-mapped receive buffer: what cudaMemcpyPeerAsync does)
  nccl     the same window as NCCL send/recv (measured before mp_init)
Predicted GB/s (mp_select t_pred) is reported next to the measured one.  One GPU per
rank (ranks whose kernels wait on one another never share a GPU).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

MiB = 1 << 20


def iters_for(n):
    return (10, 100) if n <= MiB else (4, 20) if n <= 64 * MiB else (2, 5)


def main():
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    ap = argparse.ArgumentParser()
    ap.add_argument("--min-bytes", type=int, default=4096)
    ap.add_argument("--max-bytes", type=int, default=1 << 30)
    ap.add_argument("--windows", default="1,16,64")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "omb_world.jsonl"))
    a = ap.parse_args()
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = int(os.environ.get("LOCAL_RANK", 0))
    assert torch.cuda.device_count() > dev, "one GPU per rank"
    torch.cuda.set_device(dev)
    windows = [int(w) for w in a.windows.split(",")]
    sizes = []
    n = a.min_bytes
    while n <= a.max_bytes:
        sizes.append(n)
        n *= 2
    big = sizes[-1]
    pair = rank in (0, 1)
    peer = 1 - rank if pair else None
    s_tx, s_rx = torch.cuda.Stream(), torch.cuda.Stream()
    src = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda") if pair else None
    torch.cuda.synchronize()
    out = []

    def emit(d):
        if rank == 0:
            out.append(d)
            print(json.dumps(d), flush=True)

    def gmax(x):
        t = torch.tensor([float(x)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t[0])

    # ---- NCCL send/recv windows (before mp_init: no NCCL kernel beside the engine's)
    try:
        g = dist.new_group(backend="nccl")
        rb = torch.empty(big, dtype=torch.uint8, device="cuda") if pair else None
        for n in sizes:
            skip, it = iters_for(n)
            for w in windows:
                dist.barrier()
                if pair:
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    for i in range(skip + it):
                        if i == skip:
                            e0.record()
                        ops = [dist.P2POp(dist.isend if rank == 0 else dist.irecv,
                                          src[:n] if rank == 0 else rb[:n], peer, g) for _ in range(w)]
                        for q in dist.batch_isend_irecv(ops):
                            q.wait()
                    e1.record()
                    torch.cuda.synchronize()
                    t = e0.elapsed_time(e1) * 1e-3 / it
                else:
                    t = 0.0
                t = gmax(t)
                emit({"test": "bw", "impl": "nccl", "n": n, "window": w, "GBps": n * w / t / 1e9})
        dist.destroy_process_group(g)
        del rb
        torch.cuda.synchronize()
    except Exception as exc:  # context, not the product
        emit({"impl": "nccl", "error": repr(exc)})

    ctx = mdist.context_from_dist(device=dev, calibrate=True, heap_bytes=2 * big + 64 * MiB, timeout_s=60.0)
    ctx.set_options(mode=mp.MP_MODEL_B200)
    rbuf = ctx.alloc(big) if pair else None
    ack = ctx.alloc(4096) if pair else None
    tag = [0]

    def window_bw(n, w, bidir):
        """One OMB window; returns device seconds on rank 0 (max over the pair)."""
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if pair:
            e0.record(s_tx)
            s_rx.wait_event(e0)
            for _ in range(w):
                if rank == 0 or bidir:
                    ctx.send(src, n, peer, tag[0], None, s_tx)
                if rank == 1 or bidir:
                    ctx.recv(rbuf, n, peer, tag[0], s_rx)
                tag[0] += 1
            # OMB's ack: the receiver answers with 4 bytes once the window has landed
            if rank == 1:
                s_tx.wait_stream(s_rx)
                ctx.send(src, 4, 0, 1 << 30, None, s_tx)
            else:
                s_rx.wait_stream(s_tx)
                ctx.recv(ack, 4, 1, 1 << 30, s_rx)
                s_tx.wait_stream(s_rx)
            e1.record(s_tx)
            s_tx.synchronize()
            s_rx.synchronize()
            t = e0.elapsed_time(e1) * 1e-3
        else:
            t = 0.0
        return gmax(t)

    for n in sizes:
        skip, it = iters_for(n)
        d = ctx.select(0, 1, n).as_dict()
        pred = n / d["t_pred"] / 1e9 if d["t_pred"] else None
        for w in windows:
            for bidir in (False, True):
                ts = [window_bw(n, w, bidir) for _ in range(skip + it)][skip:]
                ts.sort()
                t = ts[len(ts) // 2]
                emit({"test": "bibw" if bidir else "bw", "impl": "mp", "n": n, "window": w,
                      "GBps": n * w * (2 if bidir else 1) / t / 1e9, "pred_GBps": pred,
                      "split": [d["bytes"], d["chunks"]]})
        if n <= 4 * MiB:  # osu_latency: ping-pong
            lat = []
            for i in range(skip + it):
                dist.barrier()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                if pair:
                    e0.record(s_tx)
                    if rank == 0:
                        ctx.send(src, n, 1, tag[0], None, s_tx)
                        ctx.recv(rbuf, n, 1, tag[0] + 1, s_tx)
                    else:
                        ctx.recv(rbuf, n, 0, tag[0], s_tx)
                        ctx.send(src, n, 0, tag[0] + 1, None, s_tx)
                    e1.record(s_tx)
                    s_tx.synchronize()
                    t = e0.elapsed_time(e1) * 1e-3 / 2
                else:
                    t = 0.0
                tag[0] += 2
                t = gmax(t)
                if i >= skip:
                    lat.append(t)
            lat.sort()
            emit({"test": "latency", "impl": "mp", "n": n, "us": lat[len(lat) // 2] * 1e6})
    ctx.sync()

    # ---- copy-engine peer copy windows into the IPC-mapped receive buffer
    try:
        from cuda.bindings import runtime as rt
        offs = [None] * world
        dist.all_gather_object(offs, (rbuf - ctx.peer_base(rank)) if rbuf else None)
        for n in sizes:
            skip, it = iters_for(n)
            for w in windows:
                dist.barrier()
                t = 0.0
                if rank == 0:
                    dptr = ctx.peer_base(1) + offs[1]
                    kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    for i in range(skip + it):
                        if i == skip:
                            e0.record(s_tx)
                        for _ in range(w):
                            rt.cudaMemcpyAsync(dptr, src.data_ptr(), n, kind, s_tx.cuda_stream)
                    e1.record(s_tx)
                    s_tx.synchronize()
                    t = e0.elapsed_time(e1) * 1e-3 / it
                t = gmax(t)
                emit({"test": "bw", "impl": "ce_peer", "n": n, "window": w, "GBps": n * w / t / 1e9})
    except Exception as exc:
        emit({"impl": "ce_peer", "error": repr(exc)})

    if rank == 0:
        os.makedirs(os.path.dirname(a.out), exist_ok=True)
        with open(a.out, "w") as f:
            for d in out:
                f.write(json.dumps(d) + "\n")
    if rbuf:
        ctx.free(rbuf)
        ctx.free(ack)
    ctx.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
