"""Diagnostic: 64 KiB - 2 MiB window times with small vs 1 GiB buffers, spin-fronted,
against the banded model's prediction (why the band test's 64 KiB error varies by box)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
c = mp.Context(device=0, n_loop_relays=2, host_path=1, slot_bytes=32 * MiB, heap_bytes=16 * MiB)
c.set_options(mode=mp.MP_MODEL_B200)
c.calibrate(reps=3)
edges = [0, 64 << 10, 256 << 10, 4 * MiB, 16 * MiB, 32 * MiB, 64 * MiB, 128 * MiB]
c.calibrate_bands(edges)
s = torch.cuda.Stream()
small_s = torch.randint(0, 256, (2 * MiB,), dtype=torch.uint8, device="cuda")
small_d = torch.empty_like(small_s)
big_s = torch.randint(0, 256, (1 << 30,), dtype=torch.uint8, device="cuda")
big_d = torch.empty_like(big_s)


def window_time(dst, src, n, cfg, w=64, reps=7, sleep=4_000_000):
    ts = []
    for r in range(reps + 1):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            torch.cuda._sleep(sleep)
            e0.record(s)
            for _ in range(w):
                c.xfer(dst, src, n, cfg, s)
            e1.record(s)
        covered = not e0.query()
        e1.synchronize()
        if r:
            ts.append((e0.elapsed_time(e1) * 1e-3 / w, covered))
    ts.sort()
    return ts[len(ts) // 2]


for n in (64 << 10, 128 << 10, 256 << 10, 1 * MiB, 2 * MiB):
    cfg = c.select(0, 0, n)
    a = window_time(small_d, small_s, n, cfg)
    b = window_time(big_d, big_s, n, cfg)
    a2 = window_time(small_d, small_s, n, cfg)
    print(f"{n >> 10} KiB: pred {cfg.t_pred * 1e6:.3f} us | small {a[0] * 1e6:.3f} ({a[1]}) | big {b[0] * 1e6:.3f} "
          f"({b[1]}) | small again {a2[0] * 1e6:.3f}", flush=True)
for j, (lo, prm, port) in enumerate(c.get_model_bands(0, 0)[:4]):
    print("band", lo, "direct alpha %.3f us beta %.1f GB/s" % (prm[0]["alpha"] * 1e6, prm[0]["beta"] / 1e9))
