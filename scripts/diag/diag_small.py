#!/usr/bin/env python3
"""Where does a mid-size loopback transfer spend its time?  Back-to-back windows of
mp_xfer and cudaMemcpyAsync at 1, 8, 32 MiB (CUDA events); run it under
`ncu --metrics gpu__time_duration.sum` to get the kernel-only durations."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
from cuda.bindings import runtime as rt  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def main():
    iters = int(sys.argv[1]) if len(sys.argv) > 1 else 50
    torch.cuda.set_device(0)
    ctx = mp.Context(device=0, n_loop_relays=1, host_path=0, heap_bytes=16 * MiB)
    s = torch.cuda.Stream()
    A = torch.randint(0, 256, (32 * MiB,), dtype=torch.uint8, device="cuda")
    B = torch.empty_like(A)
    kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
    for n in (MiB, 8 * MiB, 32 * MiB):
        cfg = ctx.make_config([n, 0], [1, 0])
        for name, fn in (("mpx", lambda: ctx.xfer(B, A, n, cfg, s)),
                         ("memcpy", lambda: rt.cudaMemcpyAsync(B.data_ptr(), A.data_ptr(), n, kind, s.cuda_stream))):
            for _ in range(3):
                fn()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(iters):
                fn()
            e1.record(s)
            e1.synchronize()
            t = e0.elapsed_time(e1) * 1e3 / iters
            print(json.dumps({"n": n, "impl": name, "us_per_op": t, "GBps": n / (t * 1e-6) / 1e9}), flush=True)
    ctx.close()


if __name__ == "__main__":
    main()
