"""Design experiment (MPX_TRACE build, MPX_LIB=<it>): per-chunk timestamps of the
streamed staged lanes — the loopback relay ring alone against the emulated world's
relay path (same 16 lanes, 256 MiB, k = 16).  Per chunk: the median over lanes of
when the watcher found it ready, the publisher saw its loads land and its stores
complete, for the producer (stage-in) and the consumer (forward / relay) groups."""
import ctypes
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
n, k, lanes = 256 * MiB, 16, 16
L = mp.lib()
L.mpx_trace_set.argtypes = [ctypes.c_void_p]
tr = torch.zeros(512 * 128 * 4, dtype=torch.int64, device="cuda")
src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")


def analyse(name, groups):
    t = tr.view(512, 128, 4).cpu()
    t0 = min(int(t[c, 0, e]) for g in groups.values() for c in g for e in range(3) if int(t[c, 0, e]))
    print(f"== {name}  (µs from the first event; median over the group's lanes)")
    print("chunk " + " ".join(f"{g}:{e:>7}" for g in groups for e in ("ready", "loaded", "stored")))
    for j in range(k):
        row = []
        for g, ctas in groups.items():
            for e in range(3):
                v = [int(t[c, j, e]) for c in ctas if int(t[c, j, e])]
                row.append(f"{(statistics.median(v) - t0) / 1e3:>13.1f}" if v else f"{'-':>13}")
        print(f"{j:>5} " + " ".join(row))
    ends = [int(t[c, k - 1, 2]) for g in groups.values() for c in g if int(t[c, k - 1, 2])]
    print(f"last store {(max(ends) - t0) / 1e3:.1f} µs -> {n / ((max(ends) - t0) * 1e-9) / 1e9:.0f} GB/s")


# loopback: one relay ring, 16 lanes: CTAs 0-15 stage in, 16-31 forward
c = mp.Context(device=0, n_loop_relays=1, host_path=0, relay_ctas=lanes, heap_bytes=8 * MiB)
dst = torch.empty_like(src)
cfg = c.make_config([0, n], [1, k])
for _ in range(3):
    c.xfer(dst, src, n, cfg)
c.sync()
assert L.mpx_trace_set(tr.data_ptr()) == 0
tr.zero_()
torch.cuda.synchronize()
c.xfer(dst, src, n, cfg)
c.sync()
assert L.mpx_trace_set(None) == 0
assert torch.equal(dst, src)
nz = [i for i in range(512) if int(tr.view(512, 128, 4)[i].abs().sum())]
print("loopback CTAs with lanes:", nz)
analyse("loopback relay ring", {"prod": [i for i in nz if i < lanes], "cons": [i for i in nz if i >= lanes]})
c.close()

# emulated world 3, rank 0 -> 1 through relay rank 2 (no host path)
with mp.EmulatedWorld(3, device=0, heap_bytes=n + 64 * MiB, relay_ctas=lanes, host_path=0, timeout_s=60.0) as W:
    c0, c1 = W.ctx[0], W.ctx[1]
    d = c1.alloc(n)
    ecfg = c0.make_config([0, n], [1, k], 0, 1)
    for r in range(3):
        c0.send(src, n, 1, tag=r, cfg=ecfg)
        c1.recv(d, n, 0, tag=r)
        W.run()
    assert L.mpx_trace_set(tr.data_ptr()) == 0
    tr.zero_()
    torch.cuda.synchronize()
    c0.send(src, n, 1, tag=9, cfg=ecfg)
    c1.recv(d, n, 0, tag=9)
    print("emu grid time", W.run())
    assert L.mpx_trace_set(None) == 0
    assert torch.equal(mp.as_tensor(d, n), src)
    nz = [i for i in range(512) if int(tr.view(512, 128, 4)[i].abs().sum())]
    print("emulated CTAs with lanes:", nz)
    # grid order: receive (1 CTA, no host consumers), relay (16), gate, send (1 direct + 16 staged)
    analyse("emulated relay path", {"prod": [i for i in nz if i > 20], "cons": [i for i in nz if i <= 20 and i > 0]})
    t = tr.view(512, 128, 4).cpu()
    t0 = min(int(v) for v in t.flatten() if int(v))

    def ev(cta, j, e):
        v = int(t[cta, j, e])
        return f"{(v - t0) / 1e3:.1f}" if v else "-"
    print("start path (µs): recv CTS post", ev(0, 125, 0), "->", ev(0, 125, 1), "| gate start", ev(17, 126, 0),
          "bell write", ev(17, 126, 1), "->", ev(17, 126, 2),
          "| relay CTA 1 poll start", ev(1, 124, 0), "bell seen", ev(1, 124, 1),
          "| relay CTA 16 bell seen", ev(16, 124, 1))
