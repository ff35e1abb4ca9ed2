#!/usr/bin/env python3
"""osu_latency-style ping-pong on the multi-rank engine (torchrun, 2 ranks; both may
share one GPU under MPS — retired: ranks now get one GPU each).  Rank 0 sends n bytes to rank 1 and
waits for n bytes back; one-way latency = median round trip / 2 over `iters` (host
clock around stream-synchronised send/recv, as OSU times blocking MPI calls).
MPX_EAGER=0 forces the rendezvous protocol.  Prints JSON lines from rank 0."""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402


def main():
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    dist.init_process_group("gloo")
    rank = dist.get_rank()
    dev = int(os.environ.get("LOCAL_RANK", 0))
    assert torch.cuda.device_count() > dev, "one GPU per rank"
    torch.cuda.set_device(dev)
    s_tx, s_rx = torch.cuda.Stream(), torch.cuda.Stream()
    big = 1 << 20
    src = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    ctx = mdist.context_from_dist(device=dev, heap_bytes=16 << 20, timeout_s=30.0)
    buf = ctx.alloc(big)
    peer = 1 - rank
    ev = torch.cuda.Event()
    for n in (8, 64, 512, 4096, 16384, 65536, 262144, 1 << 20):
        iters, skip = (300, 30) if n <= 65536 else (100, 10)
        rtts = []
        dist.barrier()
        for i in range(iters + skip):
            t0 = time.perf_counter()
            if rank == 0:
                ctx.send(src, n, peer, tag=i, stream=s_tx)
                ctx.recv(buf, n, peer, tag=i, stream=s_rx)
                s_rx.synchronize()
            else:
                ctx.recv(buf, n, peer, tag=i, stream=s_rx)
                ev.record(s_rx)
                s_tx.wait_event(ev)
                ctx.send(src, n, peer, tag=i, stream=s_tx)
                s_tx.synchronize()
            if i >= skip:
                rtts.append(time.perf_counter() - t0)
        s_tx.synchronize()
        if rank == 0:
            print(json.dumps({"n": n, "eager": os.environ.get("MPX_EAGER", "1") != "0",
                              "lat_us": statistics.median(rtts) / 2 * 1e6,
                              "lat_p10_us": sorted(rtts)[len(rtts) // 10] / 2 * 1e6}), flush=True)
    ctx.sync()
    ctx.free(buf)
    ctx.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
