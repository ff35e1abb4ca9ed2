#!/usr/bin/env python3
"""Per-path timing of the multi-rank engine (torchrun, all ranks may share one GPU —
run under MPS for concurrency).  Rank 0 sends to rank 1; every config is timed over
K messages on both sides; prints JSON lines from rank 0."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

MiB = 1 << 20


def main():
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = int(os.environ.get("LOCAL_RANK", 0))
    assert torch.cuda.device_count() > dev, "one GPU per rank"
    torch.cuda.set_device(dev)
    n = int(os.environ.get("DIAG_BYTES", 64 * MiB))
    K = int(os.environ.get("DIAG_K", "20"))
    s = torch.cuda.Stream()
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    ctx = mdist.context_from_dist(device=dev, heap_bytes=n + 64 * MiB, timeout_s=30.0,
                                  calibrate=os.environ.get("DIAG_CALIBRATE", "1") == "1",
                                  relay_ctas=int(os.environ.get("DIAG_CTAS", "16")),
                                  slots=int(os.environ.get("DIAG_SLOTS", "4")))
    ps = ctx.paths(0, 1)
    buf = ctx.alloc(n) if rank == 1 else None
    cases = {"direct": ([n] + [0] * (len(ps) - 1), None)}
    hb = [0] * len(ps)
    hb[-1] = n
    kmin = -(-n // (32 * MiB - 512))  # chunks must fit the 32 MiB slots
    for k in sorted({max(kmin, k) for k in (2, 4, 8, 16)}):
        cases[f"host_k{k}"] = (hb, k)
    if world >= 3:
        rb = [0] * len(ps)
        rb[1] = n
        for k in sorted({max(kmin, k) for k in (4, 8, 16)}):
            cases[f"relay_k{k}"] = (rb, k)
    _, prm, _ = ctx.get_model(0, 1)

    def ceiling(nb):
        # the stage-group ceiling of a staged path alone: the slower of its two legs as
        # Step 1 timed them (plain copies with the stage group's CTAs)
        i = next((j for j, b in enumerate(nb) if b), 0)
        return None if i == 0 else min(prm[i]["beta"], prm[i]["beta2"]) / 1e9

    for name, (nb, kf) in cases.items():
        ks = [1] + [((kf or max(1, b // (8 * MiB))) if b else 0) for b in nb[1:]]
        cfg = ctx.make_config(nb, ks, 0, 1)
        dist.barrier()
        t0 = time.perf_counter()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for i in range(K):
            if rank == 0:
                ctx.send(src, n, 1, tag=i, cfg=cfg, stream=s)
            elif rank == 1:
                ctx.recv(buf, n, 0, tag=i, stream=s)
        e1.record(s)
        s.synchronize()
        wall = time.perf_counter() - t0
        ms = e0.elapsed_time(e1)
        out = [None] * world
        dist.all_gather_object(out, (rank, ms, wall))
        if rank == 0:
            gbs = n * K / (max(m for _, m, _ in out) * 1e-3) / 1e9
            ce = ceiling(nb)
            print(json.dumps({"case": name, "ctas": os.environ.get("DIAG_CTAS", "16"),
                              "slots": os.environ.get("DIAG_SLOTS", "4"), "bytes": nb, "chunks": ks,
                              "per_msg_ms": {r: m / K for r, m, _ in out}, "GBps": gbs,
                              "stage_group_ceiling_GBps": ce,
                              "frac_of_stage_group_ceiling": gbs / ce if ce else None}), flush=True)
    ctx.sync()
    if buf:
        ctx.free(buf)
    ctx.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
