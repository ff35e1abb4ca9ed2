"""Host-side cost per mp_xfer call from Python (ctypes) vs cudaMemcpyAsync through
cuda-python, for small messages: is the OMB small-size window loop host-bound?"""
import os, sys, time, json
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch
from cuda.bindings import runtime as rt
from paper_conf_sc_sojoodiasfga25_b200 import mp

torch.cuda.set_device(0)
ctx = mp.Context(device=0, heap_bytes=16 << 20)
ctx.set_options(mode=mp.MP_MODEL_B200)
A = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
B = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
for n in (4096, 65536, 1 << 20):
    cfg = ctx.select(0, 0, n)
    out = {"n": n}
    for name, fn in (("xfer_cfg", lambda: ctx.xfer(B, A, n, cfg, stream=s)),
                     ("xfer_sel", lambda: ctx.xfer(B, A, n, None, stream=s)),
                     ("memcpy", lambda: rt.cudaMemcpyAsync(B.data_ptr(), A.data_ptr(), n, kind, s.cuda_stream))):
        for _ in range(100):
            fn()
        s.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(s)
        for _ in range(2000):
            fn()
        t1 = time.perf_counter()
        e1.record(s)
        e1.synchronize()
        out[name + "_host_us"] = (t1 - t0) / 2000 * 1e6
        out[name + "_gpu_us"] = e0.elapsed_time(e1) * 1e3 / 2000
    print(json.dumps(out))
