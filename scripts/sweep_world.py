#!/usr/bin/env python3
"""BASELINE.json config 2 across GPUs: the static exhaustive-search distribution
(§5) against the model's dynamic pick for GPU0 -> GPU1
over the direct path and the relays GPU2, GPU3 (host path excluded, as config 2
states) — the E_sel / E_pred acceptance (C13) on the multi-rank engine.

    torchrun --nproc-per-node 4 scripts/sweep_world.py [--sizes 16,64,256] [--reps 3]
             [--step 32] [--out gpurun_out/sweep_world.json]

Grid: θ over the 3-simplex (direct, relay 2, relay 3) in steps
of 1/step, one k shared by both relays from {1, 2, 4, ..., 64} (chunks that do not
fit a 32 MiB slot are skipped), then a step-1/128 refinement around the best.  Each
config is timed as an OMB window of W back-to-back messages (median of `reps`
windows, max over the sender's and the receiver's device time); the best of the sweep
and the B200- and paper-mode picks are re-timed with 3x the repetitions.
Every rank enumerates the same configs; ranks 2.. only relay.  One GPU per rank
(ranks whose kernels wait on one another never share a GPU).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

MiB = 1 << 20
A = 256
SLOT = 32 * MiB - 512


def grid(n, step, ks, around=None, fine=128):
    """(bytes, chunks) configs over [direct, relay2, relay3] (+ host = 0)."""
    out, seen = [], set()
    if around is None:
        pts = [(i, j) for i in range(step + 1) for j in range(step + 1 - i)]
        scale = step
    else:
        scale = fine
        c1, c2 = (round(around[1] / n * fine), round(around[2] / n * fine))
        pts = [(c1 + di, c2 + dj) for di in range(-4, 5) for dj in range(-4, 5)
               if c1 + di >= 0 and c2 + dj >= 0 and c1 + di + c2 + dj <= fine]
    for a, b in pts:
        r1 = n * a // scale // A * A
        r2 = n * b // scale // A * A
        for k in (ks if (r1 or r2) else [1]):
            ok = all(r == 0 or (r // A >= k and -(-r // k) <= SLOT) for r in (r1, r2))
            if not ok:
                continue
            nb = [n - r1 - r2, r1, r2, 0]
            ch = [1, k if r1 else 0, k if r2 else 0, 0]
            key = (tuple(nb), tuple(ch))
            if key not in seen:
                seen.add(key)
                out.append((nb, ch))
    return out


def main():
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="16,64,256")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--step", type=int, default=32)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep_world.json"))
    a = ap.parse_args()
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    assert world >= 4, "config 2 needs GPU0, GPU1 and two relays"
    dev = int(os.environ.get("LOCAL_RANK", 0))
    assert torch.cuda.device_count() > dev, "one GPU per rank"
    torch.cuda.set_device(dev)
    sizes = [int(s) * MiB for s in a.sizes.split(",")]
    big = max(sizes)
    s = torch.cuda.Stream()
    src = torch.randint(0, 256, (big,), dtype=torch.uint8, device="cuda",
                        generator=torch.Generator(device="cuda").manual_seed(20251116)) if rank == 0 else None
    torch.cuda.synchronize()
    ctx = mdist.context_from_dist(device=dev, calibrate=True, heap_bytes=big + 64 * MiB, timeout_s=60.0,
                                  host_path=1)
    paths = ctx.paths(0, 1)
    assert [k for k, _ in paths][:3] == [0, 1, 1] and paths[1][1] == 2 and paths[2][1] == 3, paths
    npaths = len(paths)
    rbuf = ctx.alloc(big) if rank == 1 else None
    mask = 0b0111                                     # direct + relay 2 + relay 3 (config 2: no host)
    tag = [0]

    def measure(nb, ch, n, reps):
        """Per-message seconds: OMB window of W messages, median of reps windows."""
        W = 8 if n <= 64 * MiB else 4
        full_nb = list(nb) + [0] * (npaths - len(nb))
        full_ch = list(ch) + [0] * (npaths - len(ch))
        cfg = ctx.make_config(full_nb, full_ch, 0, 1)
        ts = []
        for _ in range(reps):
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(W):
                if rank == 0:
                    ctx.send(src, n, 1, tag[0], cfg, s)
                elif rank == 1:
                    ctx.recv(rbuf, n, 0, tag[0], s)
                tag[0] += 1
            e1.record(s)
            s.synchronize()
            ms = e0.elapsed_time(e1) if rank in (0, 1) else 0.0
            t = torch.tensor([ms], dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ts.append(float(t[0]) * 1e-3 / W)
        ts.sort()
        return ts[len(ts) // 2]

    report = {"paths": paths, "model": ctx.get_model(0, 1), "topology": ctx.topology(),
              "sizes": {}}
    ks = [1, 2, 4, 8, 16, 32, 64]
    for n in sizes:
        rows = []
        for nb, ch in grid(n, a.step, ks):
            t = measure(nb, ch, n, a.reps)
            rows.append({"bytes": nb, "chunks": ch, "t": t, "GBps": n / t / 1e9})
        coarse = max(rows, key=lambda r: r["GBps"])
        for nb, ch in grid(n, a.step, ks, around=coarse["bytes"]):
            t = measure(nb, ch, n, a.reps)
            rows.append({"bytes": nb, "chunks": ch, "t": t, "GBps": n / t / 1e9, "fine": True})
        # re-time the top 5 and the picks with more repetitions
        top = sorted(rows, key=lambda r: -r["GBps"])[:5]
        for r in top:
            r["t_final"] = measure(r["bytes"], r["chunks"], n, 3 * a.reps)
        best = max(top, key=lambda r: n / r["t_final"])
        best_bw = n / best["t_final"] / 1e9
        picks = {}
        for name, mode in (("b200", mp.MP_MODEL_B200), ("paper", mp.MP_MODEL_PAPER)):
            ctx.set_options(mode=mode)
            d = ctx.select(0, 1, n, mask).as_dict()
            t = measure(d["bytes"], d["chunks"], n, 3 * a.reps)
            bw, bwp = n / t / 1e9, n / d["t_pred"] / 1e9
            picks[name] = {"config": d, "t": t, "GBps": bw, "pred_GBps": bwp,
                           "E_sel": max(0.0, 1 - bw / best_bw), "E_pred": abs(bwp - best_bw) / best_bw}
        direct = next(r for r in rows if r["bytes"][0] == n)
        report["sizes"][str(n)] = {"best": best, "best_GBps": best_bw, "direct_only": direct, "picks": picks,
                                   "n_configs": len(rows), "rows": rows}
        if rank == 0:
            print(json.dumps({"n": n, "n_configs": len(rows), "best_GBps": best_bw,
                              "best": [best["bytes"], best["chunks"]], "direct_GBps": direct["GBps"],
                              **{f"{k}_GBps": v["GBps"] for k, v in picks.items()},
                              **{f"{k}_E_sel": v["E_sel"] for k, v in picks.items()},
                              **{f"{k}_E_pred": v["E_pred"] for k, v in picks.items()}}), flush=True)
    ctx.sync()
    if rank == 0:
        os.makedirs(os.path.dirname(a.out), exist_ok=True)
        with open(a.out, "w") as f:
            json.dump(report, f)
    if rbuf:
        ctx.free(rbuf)
    ctx.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
