#!/usr/bin/env python3
"""OSU-micro-benchmark-style sweep (BASELINE.json config 4; the paper's OMB BW/BIBW
methodology) on the single-GPU loopback engine.

    python scripts/omb.py [--min 4096] [--max 2147483648] [--out gpurun_out/omb.jsonl]

For every power-of-two size:
  bw      window w ∈ {1, 16, 64} back-to-back model-selected transfers (mp_xfer),
          GB/s = n·w / window time — next to single-path cudaMemcpyAsync (same window);
  bibw    two directions at once (A→B and B→A on two streams), GB/s counts both;
  latency one transfer, median over many (sizes ≤ 1 MiB), vs cudaMemcpyAsync.
Predicted GB/s (mp_select t_pred) is reported beside the measured one (E_pred).
Only one GPU exists in this run: NCCL send/recv and cudaMemcpyPeerAsync need two.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
from cuda.bindings import runtime as rt  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402


def timed(fn, iters, skip, stream):
    for _ in range(skip):
        fn()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(iters):
        fn()
    e1.record(stream)
    e1.synchronize()
    return e0.elapsed_time(e1) * 1e-3 / iters


def median_single(fn, reps, stream):
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e-3)
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--min", type=int, default=4096)
    ap.add_argument("--max", type=int, default=2 << 30)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "omb.jsonl"))
    ap.add_argument("--no-bands", action="store_true", help="asymptotic Step-1 model only (no NEXT f4 bands)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = mp.Context(device=0, calibrate=True, heap_bytes=16 << 20)
    ctx.set_options(mode=mp.MP_MODEL_B200)
    # predictions of the single asymptotic Hockney fit (Step 1) before the size bands
    sizes, n = [], a.min
    while n <= a.max:
        sizes.append(n)
        n *= 2
    pred_base = {n: n / ctx.select(0, 0, n).t_pred / 1e9 for n in sizes}
    if not a.no_bands:
        ctx.calibrate_bands()   # NEXT f4 (readings C20/C21)
    big = a.max
    A = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
    B = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
    # osu_bibw: each side sends from its s_buf into the peer's r_buf — the reverse
    # direction uses its own pair of buffers (a swapped A↔B pair would make each copy
    # read the lines the other is writing; profiles/r01/bibw.jsonl)
    Cb = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
    D = torch.empty(big, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    out = open(a.out, "w")
    n = a.min
    while n <= a.max:
        cfg = ctx.select(0, 0, n)
        d = cfg.as_dict()
        iters = 200 if n <= (1 << 20) else (50 if n <= (64 << 20) else 5)
        skip = 10 if n <= (64 << 20) else 2
        row = {"n": n, "config": {"bytes": d["bytes"], "chunks": d["chunks"]},
               "pred_GBps": n / d["t_pred"] / 1e9, "pred_base_GBps": pred_base[n]}
        for w in (1, 16, 64):
            def mpw():
                for _ in range(w):
                    ctx.xfer(B, A, n, None, s1)

            def cew():
                for _ in range(w):
                    rt.cudaMemcpyAsync(B.data_ptr(), A.data_ptr(), n, kind, s1.cuda_stream)
            it = max(1, iters // w) if n > (1 << 20) else max(5, iters // w)
            row[f"bw_w{w}_GBps"] = n * w / timed(mpw, it, 1, s1) / 1e9
            row[f"ce_bw_w{w}_GBps"] = n * w / timed(cew, it, 1, s1) / 1e9

        def bibw():
            ev = torch.cuda.Event()
            ev.record(s1)
            s2.wait_event(ev)
            ctx.xfer(B, A, n, None, s1)
            ctx.xfer(D, Cb, n, None, s2)
            ev2 = torch.cuda.Event()
            ev2.record(s2)
            s1.wait_event(ev2)
        row["bibw_GBps"] = 2 * n / timed(bibw, max(3, iters // 4), 2, s1) / 1e9
        if n <= (1 << 20):
            row["lat_us"] = median_single(lambda: ctx.xfer(B, A, n, None, s1), 200, s1) * 1e6
            row["ce_lat_us"] = median_single(
                lambda: rt.cudaMemcpyAsync(B.data_ptr(), A.data_ptr(), n, kind, s1.cuda_stream), 200, s1) * 1e6
        row["E_pred_w1"] = abs(row["pred_GBps"] - row["bw_w1_GBps"]) / row["bw_w1_GBps"]
        row["E_pred_base_w1"] = abs(row["pred_base_GBps"] - row["bw_w1_GBps"]) / row["bw_w1_GBps"]
        row["E_pred_w16"] = abs(row["pred_GBps"] - row["bw_w16_GBps"]) / row["bw_w16_GBps"]
        print(json.dumps(row), flush=True)
        out.write(json.dumps(row) + "\n")
        n *= 2
    ctx.sync()
    assert torch.equal(A[:1 << 20], A[:1 << 20])
    out.close()
    ctx.close()


if __name__ == "__main__":
    main()
