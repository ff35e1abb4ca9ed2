"""Design experiment (MPX_TRACE build, MPX_LIB=<it>): the multi-rank direct path's
start and end, in the emulated world: when the receiver posts its clear-to-send, when
the direct CTAs start and finish copying, when the last CTA releases the count, when
the receiver sees it.  One 16 MiB and one 256 MiB message."""
import ctypes
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20
L = mp.lib()
L.mpx_trace_set.argtypes = [ctypes.c_void_p]
tr = torch.zeros(512 * 128 * 4, dtype=torch.int64, device="cuda")
with mp.EmulatedWorld(2, device=0, heap_bytes=300 * MiB, host_path=0, timeout_s=60.0) as W:
    c0, c1 = W.ctx[0], W.ctx[1]
    for n in (16 * MiB, 256 * MiB):
        src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
        d = c1.alloc(n)
        cfg = c0.make_config([n], [1], 0, 1)
        for r in range(3):
            c0.send(src, n, 1, tag=r, cfg=cfg)
            c1.recv(d, n, 0, tag=r)
            W.run()
        assert L.mpx_trace_set(tr.data_ptr()) == 0
        tr.zero_()
        torch.cuda.synchronize()
        c0.send(src, n, 1, tag=9, cfg=cfg)
        c1.recv(d, n, 0, tag=9)
        t_grid = W.run()
        assert L.mpx_trace_set(None) == 0
        assert torch.equal(mp.as_tensor(d, n), src)
        t = tr.view(512, 128, 4).cpu()
        t0 = min(int(v) for v in t.flatten() if int(v))

        def col(j, e):
            return [(int(t[c, j, e]) - t0) / 1e3 for c in range(512) if int(t[c, j, e])]
        st, en = col(120, 0), col(120, 1)
        print(f"== {n >> 20} MiB: grid {t_grid * 1e6:.1f} µs, {len(st)} direct CTAs")
        print(f"recv CTS post {col(125, 0)} -> {col(125, 1)}; gate bells {col(126, 1)} -> {col(126, 2)}")
        print(f"direct copy start min/med/max {min(st):.1f}/{statistics.median(st):.1f}/{max(st):.1f}; "
              f"end {min(en):.1f}/{statistics.median(en):.1f}/{max(en):.1f}")
        print(f"last CTA release {col(121, 0)} -> {col(121, 1)}; receiver sees done {col(123, 0)}, fence -> {col(123, 1)}")
        c1.free(d)
