#!/usr/bin/env python3
"""One fused launch per path kind on the loopback engine, for per-kernel ncu counters
(DRAM and PCIe bytes vs duration — SURVEY §8(d)):

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,\\
pcie__read_bytes.sum,pcie__write_bytes.sum --clock-control none --csv \\
        --log-file gpurun_out/path_probe.csv python scripts/path_probe.py

Launch order (after 2 warm-ups each, so the LAST launch of each group is the one to
read): direct 1 GiB, direct 64 KiB (one-shot kernel), relay ring alone 256 MiB / 16
chunks, pinned-host path alone 256 MiB / 16 chunks, all paths (paper-mode pick,
1 GiB).  Algorithmic bytes per launch: direct 2n HBM; relay 4b HBM;
host b PCIe up + b PCIe down, 2b HBM."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB, GiB = 1 << 20, 1 << 30
torch.cuda.set_device(0)
ctx = mp.Context(device=0, n_loop_relays=6, host_path=1, heap_bytes=16 * MiB)
ps = ctx.paths()
P = len(ps)
src = torch.randint(0, 256, (GiB,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
s = torch.cuda.Stream()


def cfg_for(n, idx, k):
    nb = [0] * P
    ch = [1] + [0] * (P - 1)
    nb[idx] = n
    ch[idx] = k
    return ctx.make_config(nb, ch)


runs = [("direct_1GiB", GiB, cfg_for(GiB, 0, 1)), ("direct_64KiB", 64 << 10, cfg_for(64 << 10, 0, 1)),
        ("relay_256MiB_k16", 256 * MiB, cfg_for(256 * MiB, 1, 16)),
        ("host_256MiB_k16", 256 * MiB, cfg_for(256 * MiB, P - 1, 16))]
ctx.set_options(mode=mp.MP_MODEL_PAPER)
runs.append(("paper_pick_1GiB", GiB, ctx.select(0, 0, GiB)))
for name, n, cfg in runs:
    for _ in range(3):
        ctx.xfer(dst, src, n, cfg, s)
    s.synchronize()
    assert torch.equal(dst[:n], src[:n]), name
    print(name, cfg.as_dict()["bytes"], flush=True)
ctx.sync()
ctx.close()
