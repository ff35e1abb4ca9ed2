#!/usr/bin/env python3
"""Diagnostic: the per-message time of a stream-launched 64 KiB window (behind a
spin) on a fresh GPU, right after mp_calibrate_bands, and after a 1 GiB copy burst,
with the SM clock (NVML) at each point."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import pynvml  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
c = mp.Context(device=0, n_loop_relays=2, host_path=1, slot_bytes=32 << 20, heap_bytes=16 << 20)
c.set_options(mode=mp.MP_MODEL_B200)
src = torch.randint(0, 256, (2 << 20,), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
s = torch.cuda.Stream()
np_ = len(c.paths(0, 0))


def window(n, w=64, reps=7):
    cfg = c.make_config([n] + [0] * (np_ - 1), [1] + [0] * (np_ - 1), 0, 0)
    ts = []
    for _ in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            torch.cuda._sleep(4_000_000)
            e0.record(s)
            for _ in range(w):
                c.xfer(dst, src, n, cfg, s)
            e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3 / w)
    return sorted(ts[1:])[reps // 2]


def clk():
    return pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)


def report(tag):
    print(f"{tag:28s} 64K {window(64 << 10):.3f} us  1M {window(1 << 20):.3f} us  sm {clk()} MHz", flush=True)


report("fresh")
report("fresh again")
t0 = time.time()
c.calibrate(reps=3)
report(f"after calibrate ({time.time() - t0:.1f}s)")
t0 = time.time()
c.calibrate_bands(reps=3)
report(f"after bands ({time.time() - t0:.1f}s)")
for lo, prm, _ in c.get_model_bands(0, 0)[:2]:
    print("band", lo, "alpha %.3f us beta %.1f GB/s" % (prm[0]["alpha"] * 1e6, prm[0]["beta"] / 1e9))
cfg = c.select(0, 0, 64 << 10)
print("t_pred 64K %.3f us" % (cfg.t_pred * 1e6))
big = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
big2 = torch.empty_like(big)
t0 = time.time()
while time.time() - t0 < 5:
    big2.copy_(big)
torch.cuda.synchronize()
report("after 5 s of 1 GiB copies")
time.sleep(3)
report("after 3 s idle")
c.close() if False else None

# the C++ (Step 1) window at exactly 64 KiB: a band [64 KiB, 128 KiB] is fitted on its
# two edge samples, so its prediction at 64 KiB is that window's measurement
c2 = mp.Context(device=0, n_loop_relays=2, host_path=1, slot_bytes=32 << 20, heap_bytes=16 << 20)
c2.set_options(mode=mp.MP_MODEL_B200)
c2.calibrate(reps=3)
c2.calibrate_bands([0, 64 << 10, 128 << 10, 1 << 20], reps=5)
for n in (64 << 10, 128 << 10):
    print("Step-1 window %d B: %.3f us" % (n, c2.select(0, 0, n).t_pred * 1e6))
c = c2
print("python window 64K %.3f us, 128K %.3f us" % (window(64 << 10), window(128 << 10)))
c2.close()
