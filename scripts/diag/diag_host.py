#!/usr/bin/env python3
"""Diagnostics of the pinned-host staged path (A9) on the loopback engine: the path
alone for several chunk counts and CTA counts, against copy-engine D2H / H2D alone and
concurrently (PCIe duplex capacity).  Prints JSON lines."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def med(fn, stream, reps=5):
    ts = []
    for _ in range(reps + 1):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e-3)
    ts = sorted(ts[1:])
    return ts[len(ts) // 2]


def main():
    torch.cuda.set_device(0)
    n = 128 * MiB
    s = torch.cuda.Stream()
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
    dst = torch.empty_like(src)
    h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
    with torch.cuda.stream(s):
        t = med(lambda: h1.copy_(src, non_blocking=True), s)
    print(json.dumps({"what": "CE D2H", "GBps": n / t / 1e9}), flush=True)
    with torch.cuda.stream(s):
        t = med(lambda: dst.copy_(h1, non_blocking=True), s)
    print(json.dumps({"what": "CE H2D", "GBps": n / t / 1e9}), flush=True)
    s2 = torch.cuda.Stream()

    def both():
        e = torch.cuda.Event()
        e.record(s)
        s2.wait_event(e)
        with torch.cuda.stream(s):
            h1.copy_(src, non_blocking=True)
        with torch.cuda.stream(s2):
            dst.copy_(h2, non_blocking=True)
        e2 = torch.cuda.Event()
        e2.record(s2)
        s.wait_event(e2)
    t = med(both, s)
    print(json.dumps({"what": "CE D2H + H2D concurrently", "GBps_each": n / t / 1e9}), flush=True)
    for ctas in (8, 16, 32):
        for copy in ("bulk", "reg"):
            os.environ["MPX_COPY"] = copy
            ctx = mp.Context(device=0, n_loop_relays=1, host_path=1, relay_ctas=ctas, slot_bytes=16 * MiB,
                             heap_bytes=16 * MiB)
            ps = ctx.paths()
            for k in (1, 2, 4, 8, 16, 32):
                nb = [0] * len(ps)
                nb[-1] = n
                ks = [1] + [0] * (len(ps) - 1)
                ks[-1] = k
                if n // k > 16 * MiB - 512:
                    continue
                cfg = ctx.make_config(nb, ks)
                t = med(lambda: ctx.xfer(dst, src, n, cfg, s), s)
                print(json.dumps({"what": "host path alone", "copy": copy, "ctas": ctas, "k": k,
                                  "GBps": n / t / 1e9}), flush=True)
            ctx.sync()
            ctx.close()
    assert torch.equal(dst, src)


if __name__ == "__main__":
    main()
