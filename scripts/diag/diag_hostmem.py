#!/usr/bin/env python3
"""Is GPU access to registered (mmap + cudaHostRegister, 4 KiB pages) host memory
slower than to cudaHostAlloc'd memory?  Copy-engine and engine-kernel (TMA) D2H/H2D
bandwidth into both kinds, 64 MiB."""
import ctypes
import json
import mmap
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
from cuda.bindings import runtime as rt  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def med(fn, s, reps=7):
    ts = []
    for _ in range(reps + 1):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e-3)
    ts = sorted(ts[1:])
    return ts[len(ts) // 2]


def main():
    n = 64 * MiB
    torch.cuda.set_device(0)
    s = torch.cuda.Stream()
    dev = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
    ctx = mp.Context(device=0, n_loop_relays=1, host_path=1, heap_bytes=16 * MiB)
    ps = ctx.paths()
    cfg = ctx.make_config([n] + [0] * (len(ps) - 1), [1] + [0] * (len(ps) - 1))
    pinned = torch.empty(n, dtype=torch.uint8).pin_memory()
    m = mmap.mmap(-1, n, flags=mmap.MAP_SHARED | mmap.MAP_ANONYMOUS)
    addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
    err = rt.cudaHostRegister(addr, n, rt.cudaHostRegisterMapped | rt.cudaHostRegisterPortable)
    assert err[0] == rt.cudaError_t.cudaSuccess, err
    kinds = {"cudaHostAlloc": pinned.data_ptr(), "mmap+cudaHostRegister": addr}
    D2H, H2D = rt.cudaMemcpyKind.cudaMemcpyDeviceToHost, rt.cudaMemcpyKind.cudaMemcpyHostToDevice
    for name, hp in kinds.items():
        r = {"mem": name}
        r["ce_d2h"] = n / med(lambda: rt.cudaMemcpyAsync(hp, dev.data_ptr(), n, D2H, s.cuda_stream), s) / 1e9
        r["ce_h2d"] = n / med(lambda: rt.cudaMemcpyAsync(dev.data_ptr(), hp, n, H2D, s.cuda_stream), s) / 1e9
        r["tma_d2h"] = n / med(lambda: ctx.xfer(hp, dev, n, cfg, s), s) / 1e9
        r["tma_h2d"] = n / med(lambda: ctx.xfer(dev, hp, n, cfg, s), s) / 1e9
        print(json.dumps(r), flush=True)
    ctx.sync()
    rt.cudaHostUnregister(addr)
    ctx.close()


if __name__ == "__main__":
    main()
