"""Per-path rates of the MULTI-RANK kernels on one GPU, as an emulated world (one
cooperative grid over every rank's kernels; include/mp.h mp_emu_run).

World 3 in the engine's default launch configuration (4 slots of 32 MiB, 16 lanes per
stage group): rank 0 -> rank 1 over the direct path alone, relay rank 2 alone, the
pinned host path alone, and all three at once.  Every message is checked bit-exact
against its source.  On one GPU every path is an HBM copy (the relay path two of them,
the host path a PCIe round trip), so these are the kernels' rates, not NVLink numbers:
payload GB/s, HBM GB/s (2 B per direct / host payload byte, 4 B per relayed one) and
its fraction of MEASURED_PEAKS.json's copy bandwidth.

    python scripts/emu_perf.py [--mib 256] [--reps 7] [--out file.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mib", type=int, default=256)
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--out", default=None)
    ap.add_argument("--case", default=None, help="direct | relay | host | all (default: every case)")
    ap.add_argument("--slots", type=int, default=0, help="ring slots (default: the library's, 4)")
    ap.add_argument("--slot-mib", type=int, default=0, help="slot size in MiB (default: the library's, 32)")
    ap.add_argument("--lanes", type=int, default=16, help="CTAs per stage group (relay_ctas)")
    ap.add_argument("--chunk-mib", type=int, default=16, help="staged chunk size in MiB")
    ap.add_argument("--no-host", action="store_true", help="no pinned-host path (direct and relay cases only)")
    a = ap.parse_args()
    n = a.mib * MiB
    try:
        peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        peak = None
    torch.cuda.set_device(0)
    rows = []
    with mp.EmulatedWorld(3, device=0, heap_bytes=n + 64 * MiB, timeout_s=60.0, slots=a.slots,
                          slot_bytes=a.slot_mib * MiB, relay_ctas=a.lanes, host_path=0 if a.no_host else -1) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        assert [k for k, _ in ps] == ([0, 1] if a.no_host else [0, 1, 2])
        src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                            generator=torch.Generator(device="cuda").manual_seed(7))
        dst = c1.alloc(n)
        out = mp.as_tensor(dst, n)
        s = torch.cuda.Stream()
        q = n // 8 // 256 * 256
        cm = a.chunk_mib
        cases = {
            "direct": ([n, 0, 0], [1, 0, 0]),
            "relay": ([0, n, 0], [1, max(1, n // (cm * MiB)), 0]),
            "host": ([0, 0, n], [1, 0, max(1, n // (cm * MiB))]),
            "all": ([n - 3 * q, 2 * q, q], [1, max(1, 2 * q // (cm * MiB)), max(1, q // (cm * MiB))]),
        }
        for name, (nb, ks) in cases.items():
            if a.case and name != a.case:
                continue
            if a.no_host:
                if nb[2]:
                    continue
                nb, ks = nb[:2], ks[:2]
            ts = []
            for r in range(a.reps + 1):
                out.zero_()
                torch.cuda.synchronize()
                c0.send(src, n, 1, tag=r, cfg=c0.make_config(nb, ks, 0, 1), stream=s)
                c1.recv(dst, n, 0, tag=r, stream=s)
                t = W.run(s)
                assert torch.equal(out, src), f"{name}: payload mismatch"
                if r:
                    ts.append(t)
            t = statistics.median(ts)
            hbm = (2 * nb[0] + 4 * nb[1] + 2 * sum(nb[2:])) / t / 1e9
            row = {"case": name, "bytes": nb, "chunks": ks, "msg_bytes": n, "s_median": t,
                   "s_min": min(ts), "payload_GBps": n / t / 1e9, "hbm_GBps": hbm,
                   "hbm_frac": hbm / peak if peak else None, "lanes": a.lanes, "slots": a.slots,
                   "slot_mib": a.slot_mib,
                   "note": "one GPU: every path is an HBM copy; not NVLink evidence"}
            rows.append(row)
            print(json.dumps(row), flush=True)
        c1.free(dst)
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
