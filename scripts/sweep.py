#!/usr/bin/env python3
"""Static exhaustive-search distribution (§5) vs the model's pick
 on the single-GPU loopback engine: the E_sel / E_pred acceptance numbers
(C13).

    python scripts/sweep.py [--sizes 16,64,256,1024] [--reps 7] [--out gpurun_out/sweep.json]

For every size the sweep measures a grid of configs — θ_host, θ shared by the
first r relays (r in {0,1,2,6}), one k for the relays and one for the host — plus the
B200-mode and the paper-mode picks of mp_select, each the median of `reps` CUDA-event
timings of one fused launch.  E_sel = 1 − BW(model pick)/BW(best of sweep);
E_pred = |BW_pred − BW_best|/BW_best.
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def measure(ctx, dst, src, n, cfg, reps, stream):
    """OMB-style (reading C21): a window of W back-to-back transfers of
    the config, seconds per message = window time / W, median over `reps` windows."""
    # windows as Step 1 times its bands (C21): long enough that the events and the first
    # launch around a window (~2-3 µs) stay a small part of it
    W = 64 if n <= 4 * MiB else 16 if n <= 64 * MiB else 2
    ts = []
    for r in range(reps + 1):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        # a ~1 ms spin kernel first, so that the whole window is enqueued before the
        # GPU reaches it: the window is then timed at GPU speed, not at the Python
        # loop's (a back-to-back 16 MiB message takes ~4 µs under PDL)
        with torch.cuda.stream(stream):
            torch.cuda._sleep(2_000_000)
        e0.record(stream)
        for _ in range(W):
            ctx.xfer(dst, src, n, cfg, stream)
        e1.record(stream)
        e1.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1) * 1e-3 / W)
    ts.sort()
    return ts[len(ts) // 2]


def grid(n, npaths, host_idx):
    A = 256
    out = []
    relay_sets = [0, 1, 2, 6]
    th_relay = [0, 1 / 64, 1 / 32, 1 / 16, 1 / 8]
    th_host = [0, 1 / 512, 1 / 256, 1 / 128, 1 / 64, 1 / 32]
    ks = [1, 2, 4, 8]
    for r, tr, th, kr, kh in itertools.product(relay_sets, th_relay, th_host, ks, ks):
        if (r == 0) != (tr == 0):
            continue
        if r == 0 and kr != 1:
            continue
        if th == 0 and kh != 1:
            continue
        nb = [0] * npaths
        ch = [1] + [0] * (npaths - 1)
        for i in range(1, 1 + r):
            nb[i] = int(n * tr) // A * A
            ch[i] = kr
        nb[host_idx] = int(n * th) // A * A
        ch[host_idx] = kh if nb[host_idx] else 0
        for i in range(1, npaths):
            if nb[i] == 0:
                ch[i] = 0
            elif nb[i] // A < ch[i] or nb[i] // ch[i] > 30 * MiB:
                break
        else:
            nb[0] = n - sum(nb)
            if nb[0] >= 0:
                out.append((nb, ch))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="16,64,256,1024")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.json"))
    ap.add_argument("--no-bands", action="store_true", help="skip the size-band picks (NEXT f4)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = mp.Context(device=0, calibrate=True, n_loop_relays=6, host_path=1, heap_bytes=16 * MiB)
    paths = ctx.paths()
    host_idx = len(paths) - 1
    stream = torch.cuda.Stream()
    sizes = [int(s) * MiB for s in a.sizes.split(",")]
    big = max(sizes)
    src = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
    dst = torch.empty(big, dtype=torch.uint8, device="cuda")
    report = {"paths": paths, "model": ctx.get_model(0, 0), "sizes": {}}
    for n in sizes:
        rows = []
        for nb, ch in grid(n, len(paths), host_idx):
            t = measure(ctx, dst, src, n, ctx.make_config(nb, ch), a.reps, stream)
            rows.append({"bytes": nb, "chunks": ch, "t": t, "GBps": n / t / 1e9})
        best = max(rows, key=lambda r: r["GBps"])
        picks = {}
        for name, mode in (("b200", mp.MP_MODEL_B200), ("paper", mp.MP_MODEL_PAPER)):
            ctx.set_options(mode=mode)
            cfg = ctx.select(0, 0, n)
            t = measure(ctx, dst, src, n, cfg, a.reps, stream)
            d = cfg.as_dict()
            bw, bwp = n / t / 1e9, n / d["t_pred"] / 1e9
            picks[name] = {"config": d, "t": t, "GBps": bw, "pred_GBps": bwp,
                           "E_sel": max(0.0, 1 - bw / best["GBps"]),
                           "E_pred": abs(bwp - best["GBps"]) / best["GBps"]}
        direct = next(r for r in rows if r["bytes"][0] == n)
        assert torch.equal(dst[:n], src[:n])
        report["sizes"][str(n)] = {"best": best, "direct_only": direct, "picks": picks, "n_configs": len(rows),
                                   "rows": rows}
        print(json.dumps({"n": n, "best_GBps": best["GBps"], "best": [best["bytes"], best["chunks"]],
                          "direct_GBps": direct["GBps"],
                          **{f"{k}_GBps": v["GBps"] for k, v in picks.items()},
                          **{f"{k}_E_sel": v["E_sel"] for k, v in picks.items()},
                          **{f"{k}_E_pred": v["E_pred"] for k, v in picks.items()}}), flush=True)
    if not a.no_bands:
        # NEXT f4 (readings C20/C21): the B200-mode pick with per-band Step-1 parameters
        ctx.calibrate_bands()
        report["bands"] = ctx.get_model_bands(0, 0)
        ctx.set_options(mode=mp.MP_MODEL_B200)
        for n in sizes:
            rs = report["sizes"][str(n)]
            cfg = ctx.select(0, 0, n)
            t = measure(ctx, dst, src, n, cfg, a.reps, stream)
            d = cfg.as_dict()
            bw, bwp = n / t / 1e9, n / d["t_pred"] / 1e9
            best = rs["best"]["GBps"]
            rs["picks"]["b200_bands"] = {"config": d, "t": t, "GBps": bw, "pred_GBps": bwp,
                                         "E_sel": max(0.0, 1 - bw / best), "E_pred": abs(bwp - best) / best}
            print(json.dumps({"n": n, "b200_bands_GBps": bw, "b200_bands_E_sel": rs["picks"]["b200_bands"]["E_sel"],
                              "b200_bands_E_pred": rs["picks"]["b200_bands"]["E_pred"]}), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(report, f)
    ctx.close()


if __name__ == "__main__":
    main()
