#!/usr/bin/env python3
"""Pinned-host path (A9) design sweep on the loopback engine: SM-driven PCIe legs with
the full direct grid (device→host writes, host→device reads, both at once) against the
copy engine, then the staged host path alone over stage-group CTA counts, chunk
counts, slot sizes and copy modes.  Prints JSON lines."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
n = 256 * MiB


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


def out(**kw):
    print(json.dumps(kw), flush=True)


torch.cuda.set_device(0)
s, s2 = torch.cuda.Stream(), torch.cuda.Stream()
src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
h2.copy_(src.cpu())


def both(f1, f2):
    def run():
        e = torch.cuda.Event()
        e.record(s)
        s2.wait_event(e)
        f1(s)
        f2(s2)
        e2 = torch.cuda.Event()
        e2.record(s2)
        s.wait_event(e2)
    return run


t = med(lambda: h1.copy_(src, non_blocking=True), s) if False else None
with torch.cuda.stream(s):
    out(what="CE D2H", GBps=n / med(lambda: h1.copy_(src, non_blocking=True), s) / 1e9)
    out(what="CE H2D", GBps=n / med(lambda: dst.copy_(h2, non_blocking=True), s) / 1e9)


def ce_d2h(st):
    with torch.cuda.stream(st):
        h1.copy_(src, non_blocking=True)


def ce_h2d(st):
    with torch.cuda.stream(st):
        dst.copy_(h2, non_blocking=True)


out(what="CE D2H + H2D concurrently", GBps_each=n / med(both(ce_d2h, ce_h2d), s) / 1e9)

for mode in ("bulk", "reg"):
    os.environ["MPX_COPY"] = "reg" if mode == "reg" else "tma"
    ctx = mp.Context(device=0, n_loop_relays=0, host_path=0, heap_bytes=16 * MiB)
    P = len(ctx.paths())
    cfg = ctx.make_config([n] + [0] * (P - 1), [1] + [0] * (P - 1))
    out(what="SM direct D2H (full grid)", copy=mode,
        GBps=n / med(lambda: ctx.xfer(h1.data_ptr(), src, n, cfg, s), s) / 1e9)
    out(what="SM direct H2D (full grid)", copy=mode,
        GBps=n / med(lambda: ctx.xfer(dst, h2.data_ptr(), n, cfg, s), s) / 1e9)
    out(what="SM direct D2H + H2D concurrently", copy=mode,
        GBps_each=n / med(both(lambda st: ctx.xfer(h1.data_ptr(), src, n, cfg, st),
                               lambda st: ctx.xfer(dst, h2.data_ptr(), n, cfg, st)), s) / 1e9)
    ctx.close()
    for ctas in (8, 16, 32):
        for slot_mib in (8, 32):
            ctx = mp.Context(device=0, n_loop_relays=0, host_path=1, heap_bytes=16 * MiB, relay_ctas=ctas,
                             slot_bytes=slot_mib * MiB)
            P = len(ctx.paths())
            for k in (8, 16, 32, 64):
                if n // k > slot_mib * MiB - 512:
                    continue
                cfg = ctx.make_config([0] * (P - 1) + [n], [1] + [0] * (P - 2) + [k])
                t = med(lambda: ctx.xfer(dst, src, n, cfg, s), s)
                out(what="host path alone", copy=mode, ctas=ctas, slot_MiB=slot_mib, k=k, GBps=n / t / 1e9)
            ctx.sync()
            assert torch.equal(dst, src)
            ctx.close()
