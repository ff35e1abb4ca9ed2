#!/usr/bin/env python3
"""Design experiment (tooling): one relay ring alone on the loopback engine, 256 MiB,
over chunk counts, ring slots and stage-group sizes; GB/s against the ring's
stage-group ceiling (the slower leg as a plain copy with the same CTAs, Step 1)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
n = 256 * MiB
src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
s = torch.cuda.Stream()


def med(fn, reps=7):
    ts = []
    for _ in range(reps + 1):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            torch.cuda._sleep(100_000)
        a.record(s)
        fn()
        b.record(s)
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e-3)
    return sorted(ts[1:])[reps // 2]


for ctas in (8, 16, 32):
    for slots, slot_mib in ((4, 32), (8, 16), (16, 8)):
        c = mp.Context(device=0, n_loop_relays=1, host_path=0, slots=slots, slot_bytes=slot_mib * MiB,
                       relay_ctas=ctas, heap_bytes=8 * MiB)
        lp = c.get_model(0, 0)[1][1]
        ceil_ = min(lp["beta"], lp["beta2"]) / 1e9
        for k in (8, 16, 32, 64):
            if n // k > slot_mib * MiB - 512:
                continue
            cfg = c.make_config([0, n], [1, k])
            t = med(lambda: c.xfer(dst, src, n, cfg, s))
            print(json.dumps(dict(ctas=ctas, slots=slots, slot_mib=slot_mib, k=k, GBps=n / t / 1e9,
                                  ceiling_GBps=ceil_, frac=n / t / 1e9 / ceil_)), flush=True)
        c.sync()
        assert torch.equal(dst, src)
        c.close()
