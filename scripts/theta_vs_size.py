#!/usr/bin/env python3
"""θ(n): the share of every path chosen by mp_select, per message size (the analogue
of the paper's Figure 4), in PAPER and B200 mode.  CPU only
(model-only contexts).

Two parameter sets:
  * loopback: the model Step 1 calibrated on one B200 (profiles/r01/calibrated_params.txt);
  * nvswitch (illustrative, not measured): an 8-GPU NVSwitch node as the model sees a
    pair — direct NVLink α 2 µs / β 750 GB/s, six relays with the same legs and ε 1.5 µs,
    a PCIe Gen5 host path (α 5 µs, β 52 / 50 GB/s, ε 3 µs), the source egress port
    shared by all NVLink paths (β 900 GB/s).

    python scripts/theta_vs_size.py [--out profiles/r01/theta_vs_size.jsonl]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_sojoodiasfga25_b200 import mp  # noqa: E402

MiB = 1 << 20


def nvswitch(c):
    paths = [(mp.MP_PATH_DIRECT, -1)] + [(mp.MP_PATH_GPU, r) for r in range(2, 8)] + [(mp.MP_PATH_HOST, -1)]
    prm = [dict(alpha=2e-6, beta=750e9, w=1.0)]
    prm += [dict(alpha=2e-6, beta=750e9, alpha2=2e-6, beta2=750e9, eps=1.5e-6, c=1.0, w=1.0) for _ in range(6)]
    prm += [dict(alpha=5e-6, beta=52e9, alpha2=5e-6, beta2=50e9, eps=3e-6, c=1.0, w=0.0)]
    c.set_model(0, 1, paths, prm, dict(alpha=2e-6, beta=900e9))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r01", "theta_vs_size.jsonl"))
    a = ap.parse_args()
    sizes = [1 << s for s in range(21, 32)]  # 2 MiB .. 2 GiB
    rows = []
    for name in ("loopback", "nvswitch"):
        for mode, mname in ((mp.MP_MODEL_PAPER, "paper"), (mp.MP_MODEL_B200, "b200")):
            world = 1 if name == "loopback" else 8
            with mp.Context(world=world, rank=0, model_only=True) as c:
                if name == "loopback":
                    c.load_params(os.path.join(ROOT, "profiles", "r01", "calibrated_params.txt"))
                    src, dst = 0, 0
                else:
                    nvswitch(c)
                    src, dst = 0, 1
                c.set_options(mode=mode, slot_bytes=32 * MiB - 512)
                kinds = c.paths(src, dst)
                for n in sizes:
                    d = c.select(src, dst, n).as_dict()
                    rows.append(dict(params=name, mode=mname, n=n, paths=kinds,
                                     theta=[b / n for b in d["bytes"]], chunks=d["chunks"],
                                     pred_GBps=n / d["t_pred"] / 1e9))
    with open(a.out, "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    for r in rows:
        th = r["theta"]
        print(f"{r['params']:9s} {r['mode']:5s} {r['n'] >> 20:5d} MiB direct {th[0]:.3f} relays "
              f"{sum(th[1:-1]):.3f} host {th[-1]:.3f}  {r['pred_GBps']:8.1f} GB/s")


if __name__ == "__main__":
    main()
