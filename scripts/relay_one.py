#!/usr/bin/env python3
"""Profiling target (tooling): one loopback relay ring alone, 256 MiB, k chunks,
RELAY_CTAS lanes — a few launches for ncu (-k regex:xfer_kernel)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
n = int(os.environ.get("RELAY_BYTES", 256 * MiB))
k = int(os.environ.get("RELAY_K", 16))
src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
c = mp.Context(device=0, n_loop_relays=1, host_path=0, relay_ctas=int(os.environ.get("RELAY_CTAS", 16)),
               heap_bytes=8 * MiB)
cfg = c.make_config([0, n], [1, k])
for _ in range(int(os.environ.get("RELAY_REPS", 4))):
    c.xfer(dst, src, n, cfg)
c.sync()
assert torch.equal(dst, src)
c.close()
print("ok")
