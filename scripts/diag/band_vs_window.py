#!/usr/bin/env python3
"""Diagnostic: the size-band model's direct-only prediction against the sweep's own
window timing (scripts/sweep.py: measure) at 4-256 MiB on the loopback engine."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402
from sweep import measure  # noqa: E402

MiB = 1 << 20
ctx = mp.Context(calibrate=True)
ctx.set_options(mode=mp.MP_MODEL_B200)
ctx.calibrate_bands()
big = 256 * MiB
src = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
s = torch.cuda.Stream()
np_ = len(ctx.paths(0, 0))
for mib in (1 / 16, 1 / 4, 1, 2, 4, 6, 8, 12, 16, 24, 32, 40, 48, 56, 64, 96, 128, 256):
    n = int(mib * MiB)
    cfg = ctx.make_config([n] + [0] * (np_ - 1), [1] + [0] * (np_ - 1), 0, 0)
    t_pred = ctx.predict(0, 0, n, cfg)
    t = measure(ctx, dst, src, n, cfg, 7, s)
    print(f"{mib:7.3f} MiB  pred {n / t_pred / 1e9:8.1f} GB/s  sweep window {n / t / 1e9:8.1f} GB/s  "
          f"err {abs(t_pred - t) / t * 100:5.1f} %", flush=True)
for lo, prm, port in ctx.get_model_bands(0, 0):
    print("band", lo // 1024, "KiB  direct alpha %.2f us beta %.1f GB/s" % (prm[0]["alpha"] * 1e6, prm[0]["beta"] / 1e9))
ctx.close()
