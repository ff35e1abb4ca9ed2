#!/usr/bin/env python3
"""Diagnostic: per-message time of stream-launched direct-only windows, 4 KiB - 4 MiB."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

c = mp.Context(device=0, n_loop_relays=2, host_path=1, slot_bytes=32 << 20, heap_bytes=16 << 20)
src = torch.randint(0, 256, (4 << 20,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
s = torch.cuda.Stream()
np_ = len(c.paths(0, 0))
for n in [4 << 10 << i for i in range(11)] + [48 << 10, 96 << 10, 192 << 10]:
    cfg = c.make_config([n] + [0] * (np_ - 1), [1] + [0] * (np_ - 1), 0, 0)
    ts = []
    for _ in range(8):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            torch.cuda._sleep(4_000_000)
            e0.record(s)
            for _ in range(64):
                c.xfer(dst, src, n, cfg, s)
            e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3 / 64)
    print(f"{n >> 10:6d} KiB  {sorted(ts[1:])[3]:.3f} us", flush=True)

# Step 1's own windows at the same sizes: one band per sample interval, so the band at
# e_j predicts exactly the window Step 1 measured at e_j
edges = [0] + [4 << 10 << i for i in range(11)]
c.calibrate(reps=3)
c.calibrate_bands(edges, reps=7)
for n in edges[1:]:
    print(f"step1 {n >> 10:6d} KiB  {c.select(0, 0, n).t_pred * 1e6:.3f} us", flush=True)
c.calibrate_bands([0, 256 << 10, 4 << 20], reps=7)
for n in (4 << 10, 16 << 10, 64 << 10, 256 << 10):
    print(f"band[0,256K) fit {n >> 10:6d} KiB  {c.select(0, 0, n).t_pred * 1e6:.3f} us", flush=True)
