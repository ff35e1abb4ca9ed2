#!/usr/bin/env python3
"""Benchmark of the multi-path P2P hot path (BASELINE.json metric:
"P2P GB/s vs msg size (% of path roofline); model-vs-sweep optimum error %").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mpx|reference]
                    [--size BYTES] [--mode b200|paper] [--workload config3|config5]

One *step* = one message through the whole hot path: mp_select (Alg 1, cached after
the first call — §8(a) A1-A6) and the transfer launches (A7 direct, A8 relays, A9
pinned-host PCIe, A10 completion).

N = 1 (default): BASELINE.json config 3 — 1 GiB, direct + 6 relays + pinned host —
on the single-GPU loopback engine (the relay rings stand in for the intermediate
GPUs; the host leg is real PCIe); the config is the B200-mode model's pick after an
init-time calibration (Step 1).  Inputs are 1 GiB (> 126 MB L2), so no flush.
config.selected names the split that executed.
N > 1 (torchrun): config 3 proper — one 1 GiB message GPU0 → GPU1 over the direct
NVLink path, the relays GPU2..GPU{N-1} and the pinned-host path ("scaling":
"strong"; value = GPU0→GPU1 payload GB/s, max-over-ranks device time), with NCCL
send/recv and copy-engine peer-copy baselines on the same pair, every path alone,
and the roofline against the source GPU's NVLink egress + PCIe.  --workload
config5: disjoint pairs (2i ↔ 2i+1) exchanging 256 MiB each way, every GPU busy.

--impl reference: the CPU oracle (oracle/, fp64 model + memcpy replay) on a bounded
sample of the same workload, one piece per host core, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

GiB, MiB = 1 << 30, 1 << 20
METRIC = "P2P GB/s vs msg size (% of path roofline); model-vs-sweep optimum error %"


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class Clocks:
    """Sample SM clocks and clock-event (throttle) reasons during the timed region via
    NVML (the same counters nvidia-smi reports), every 20 ms; falls back to one
    nvidia-smi query per sample if NVML is unavailable."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4}

    def __init__(self, index=0):
        self.index, self.samples, self.stop_ = index, [], threading.Event()
        self.t = threading.Thread(target=self._run, daemon=True)
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _sample(self):
        if self.nv is not None:
            sm = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
            try:
                mask = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                mask = self.nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
            return float(sm), int(mask)
        out = subprocess.run(["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm",
                              "--format=csv,noheader,nounits"], capture_output=True, text=True,
                             timeout=5).stdout.strip().split(",")
        self.max_mhz = float(out[1])
        return float(out[0]), 0

    def _run(self):
        while not self.stop_.is_set():
            try:
                self.samples.append(self._sample())
            except Exception:
                pass
            self.stop_.wait(0.02)

    def __enter__(self):
        try:
            self.samples.append(self._sample())
        except Exception:
            pass
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop_.set()
        self.t.join(timeout=10)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        sm = sorted(s[0] for s in self.samples)
        reasons = sorted({n for _, m in self.samples for n, bit in self.REASONS.items() if m & bit})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(self.samples), "source": "nvml" if self.nv is not None else "nvidia-smi"}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def hbm_bytes(d):
    """Algorithmic HBM bytes of one loopback message: every payload
    byte is read once from src and written once to dst; a relay byte is also written
    to and read from its ring slot; a host byte's slot traffic is PCIe/host DRAM."""
    paths, nb = d["paths"], d["bytes"]
    relay = sum(b for (k, _), b in zip(paths, nb) if k == 1)
    return 2 * sum(nb) + 2 * relay


def host_cpu():
    """(threads this process may run on, CPU model) of the host."""
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return cores, model


def _oracle_split(cfg_d, sample, n):
    """The selected split scaled to a sample of `sample` bytes (same θ, same k)."""
    scale = sample / n
    nb = [int(b * scale) // 256 * 256 for b in cfg_d["bytes"]]
    nb[0] += sample - sum(nb)
    ch = [max(1, min(c, max(1, b // 256))) if b else 0 for b, c in zip(nb, cfg_d["chunks"])]
    ch[0] = 1
    return nb, ch


def cpu_oracle_run(n, cfg_d, params, budget_s=8.0, sample=256 * MiB):
    """Time the oracle as it stands (fp64 Alg 1 select + numpy memcpy replay through the
    split; never tuned) on a bounded sample of the workload: single-threaded, then on
    every host core (the sample cut into one piece per core, each piece replayed by
    its own thread through the same split — numpy releases the GIL in the copies).
    Returns the cpu_baseline dict (value = the all-core rate)."""
    import numpy as np
    from concurrent.futures import ThreadPoolExecutor

    import synth
    from oracle import model as OM
    from oracle import transfer as OX
    kinds = [k for k, _ in cfg_d["paths"]]
    paths = [OM.Path(kind=k, via=v, **{f: (p[f] if not (k == 0 and f == "beta2") else float("inf"))
                                        for f in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")})
             for (k, v), p in zip(cfg_d["paths"], params)]
    cores, model = host_cpu()

    def rate(threads):
        piece = sample // threads // 256 * 256
        nb, ch = _oracle_split(cfg_d, piece, n)
        srcs = [synth.payload(piece, t) for t in range(threads)]
        dsts = [np.zeros(piece, dtype=np.uint8) for _ in range(threads)]

        def one(t):
            OM.select(piece, paths, OM.Options(mode=OM.B200))
            OX.replay(srcs[t], nb, ch, kinds, 256, dsts[t])

        with ThreadPoolExecutor(threads) as ex:
            list(ex.map(one, range(threads)))          # warm (page faults)
            t0 = time.perf_counter()
            reps = 0
            while True:
                list(ex.map(one, range(threads)))
                reps += 1
                if time.perf_counter() - t0 > budget_s / 2 or reps >= 50:
                    break
            dt = time.perf_counter() - t0
        assert all(np.array_equal(d, s_) for d, s_ in zip(dsts, srcs))
        return piece * threads * reps / dt / 1e9, reps, piece

    v1, r1, p1 = rate(1)
    vN, rN, pN = rate(cores) if cores > 1 else (v1, r1, p1)
    return {"value": vN, "unit": "GB/s", "cores": cores, "kind": "oracle",
            "sample": f"all cores: {rN} x {cores} pieces of {pN >> 20} MiB; single thread: {r1} x {p1 >> 20} MiB; "
                      f"each piece the {n >> 20} MiB split scaled (same θ, k), fp64 select + numpy replay",
            "single_thread_GBps": v1, "cpu_model": model}


def run_reference(args):
    """--impl reference: the CPU oracle as it stands (fp64 Alg 1 + numpy memcpy replay of
    the config-3 split), one bounded sample per step cut into one piece per host core
    (a thread each), rank 0 only."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import numpy as np
    from concurrent.futures import ThreadPoolExecutor

    import synth
    from oracle import model as OM
    from oracle import transfer as OX
    n = args.size
    tbl = synth.topology(0, 6, True)
    paths = [OM.Path(**t) for t in tbl]
    opts = OM.Options(mode=OM.B200 if args.mode == "b200" else OM.PAPER, slot_bytes=32 * MiB - 512)
    cfg = OM.select(n, paths, opts, OM.Port(4e-6, 6.5e12))
    cores, model = host_cpu()
    sample = min(n, 32 * MiB)
    piece = sample // cores // 256 * 256
    nb, ch = _oracle_split({"bytes": cfg.bytes, "chunks": cfg.chunks}, piece, n)
    kinds = [t["kind"] for t in tbl]
    srcs = [synth.payload(piece, t) for t in range(cores)]
    dsts = [np.zeros(piece, dtype=np.uint8) for _ in range(cores)]

    def one(t):
        OM.select(piece, paths, opts, OM.Port(4e-6, 6.5e12))
        OX.replay(srcs[t], nb, ch, kinds, 256, dsts[t])

    with ThreadPoolExecutor(cores) as ex:
        def step():
            list(ex.map(one, range(cores)))

        for _ in range(args.warmup):
            step()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            step()
        dt = time.perf_counter() - t0
    assert all(np.array_equal(d, s_) for d, s_ in zip(dsts, srcs))
    v = piece * cores * args.steps / dt / 1e9
    desc = (f"{cores} pieces x {piece >> 20} MiB per step (one thread per host core) of the {n >> 20} MiB "
            f"config-3 split (numpy memcpy replay + fp64 select)")
    line = {"metric": METRIC, "value": v, "unit": "GB/s", "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak" if world == 1 else "strong", "vs_baseline": None,
            "dtype": "u8", "data": "synthetic", "config": workload_config(args, world),
            "cpu_baseline": {"value": v, "unit": "GB/s", "cores": cores, "kind": "oracle", "sample": desc,
                             "cpu_model": model},
            "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def split_label(d):
    """The executed split in words, e.g. "direct-only" or
    "direct 61.2% + relays 2,3 38.8% (k 8,8)"."""
    n = sum(d["bytes"]) or 1
    used = [(k, v, b, c) for (k, v), b, c in zip(d["paths"], d["bytes"], d["chunks"]) if b]
    if len(used) == 1 and used[0][0] == 0:
        return "direct-only"
    parts = []
    for kind, name in ((0, "direct"), (1, "relays"), (2, "host")):
        sel = [(v, b, c) for k, v, b, c in used if k == kind]
        if not sel:
            continue
        share = 100.0 * sum(b for _, b, _ in sel) / n
        if kind == 0:
            parts.append(f"direct {share:.1f}%")
        elif kind == 1:
            parts.append(f"relays {','.join(str(v) for v, _, _ in sel)} {share:.1f}% "
                         f"(k {','.join(str(c) for _, _, c in sel)})")
        else:
            parts.append(f"host {share:.1f}% (k {sel[0][2]})")
    return " + ".join(parts)


def workload_config(args, world, d=None):
    if world > 1 and args.workload == "config5":
        return {"workload": f"config5 (disjoint pairs, both directions): {world // 2} pairs 2i<->2i+1, "
                            f"{args.size >> 20} MiB per message, direct + relays + pinned host, model-selected",
                "msg_bytes": args.size, "mode": args.mode, "parallelism": f"pairs{world // 2}x2dir",
                "selected": split_label(d) if d else None,
                "l2": "messages >= 126 MB L2 (no flush)" if args.size >= 128 * MiB else "no flush"}
    if world > 1:
        return {"workload": f"config3: {args.size >> 20} MiB GPU0->GPU1, direct + relays GPU2..GPU{world - 1} "
                            f"+ pinned-host PCIe, {args.mode}-mode model-selected split"
                            if world > 2 else
                            f"config3 at N=2: {args.size >> 20} MiB GPU0->GPU1, direct + pinned-host PCIe "
                            f"(no relay GPU), {args.mode}-mode model-selected split",
                "msg_bytes": args.size, "mode": args.mode, "paths": f"direct+{world - 2}relay+host",
                "selected": split_label(d) if d else None,
                "parallelism": f"p2p-1pair+{world - 2}relays",
                "l2": "message 1 GiB > 126 MB L2 (no flush)" if args.size >= 128 * MiB else "no flush"}
    return {"workload": "config3: 1 GiB GPU0->GPU0 loopback, direct + 6 relay rings + pinned-host PCIe, "
                        "B200-mode model-selected split" if args.size == GiB else
            f"{args.size} B loopback, direct + 6 relay rings + pinned host, model-selected",
            "msg_bytes": args.size, "mode": args.mode, "paths": "direct+6relay+host (available)",
            "selected": split_label(d) if d else None,
            "l2": "inputs 1 GiB > 126 MB L2 (no flush)", "parallelism": f"replicas{world}"}


def esel_grid(n, npaths, host_idx):
    """The bench's compact exhaustive sweep (scripts/sweep.py: grid, reduced): θ shared
    by the first r relays (r in {0, 1, all}), θ_host, one k for the relays and one for
    the host; the direct path takes the rest."""
    A = 256
    out = []
    for r in (0, 1, npaths - 2):
        for tr in ((0,) if r == 0 else (1 / 64, 1 / 16)):
            for th in (0, 1 / 256, 1 / 64):
                for kr in ((1,) if r == 0 else (1, 4)):
                    for kh in ((1,) if th == 0 else (1, 4)):
                        nb, ch = [0] * npaths, [1] + [0] * (npaths - 1)
                        for i in range(1, 1 + r):
                            nb[i], ch[i] = int(n * tr) // A * A, kr
                        if th:
                            nb[host_idx], ch[host_idx] = int(n * th) // A * A, kh
                        if any(nb[i] and nb[i] // ch[i] > 30 * MiB for i in range(1, npaths)):
                            continue
                        nb[0] = n - sum(nb)
                        out.append((nb, ch))
    return out


def rank_device(local, world):
    """The GPU of this rank: one per rank (device LOCAL_RANK, or device 0 when the
    launcher shows each rank only its own GPU), checked by all-gathering the GPUs'
    UUIDs.  Ranks whose kernels wait on one another are never separate launches sharing
    a GPU (B200 profiling guide); the one-GPU stand-in for the multi-rank engine is the
    emulated world (tests/test_emulated_gpu.py).  Needs the process group."""
    import torch
    import torch.distributed as dist
    n = torch.cuda.device_count()
    dev = local if local < n else 0
    uuid = str(torch.cuda.get_device_properties(dev).uuid) if n else ""
    uuids = [None] * world
    dist.all_gather_object(uuids, uuid)
    if not n or len(set(uuids)) != world:
        raise SystemExit(f"bench.py --gpus {world}: needs one GPU per rank; this node gives the ranks "
                         f"{len(set(u for u in uuids if u))} distinct GPU(s)")
    return dev


def p2p_roles(world):
    """Config 3 on N GPUs (BASELINE.json configs[2]; P:352's 2_GPUs / 3_GPUs setups):
    rank 0 sends one message to rank 1; ranks 2..N-1 are the relay GPUs; the host
    path is the pinned-host PCIe path."""
    return ["sender" if r == 0 else "receiver" if r == 1 else "relay" for r in range(world)]


def p2p_plan(ctx, world, n, mode):
    """Roles and the model's config for config 3 (every rank computes the same)."""
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    ctx.set_options(mode=mp.MP_MODEL_B200 if mode == "b200" else mp.MP_MODEL_PAPER)
    return p2p_roles(world), ctx.select(0, 1, n)


def run_world(args, world, rank, local):
    if args.workload == "config5":
        return run_world_pairs(args, world, rank, local)
    return run_world_p2p(args, world, rank, local)


def _gather_max(x):
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t[0])


def _gather_sum(x):
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t[0])


def run_world_p2p(args, world, rank, local):
    """N > 1 (torchrun, one process per GPU), the primary multi-GPU line: BASELINE.json
    config 3 — one message of --size bytes (default 1 GiB) from GPU0 to GPU1, split by
    the model (Alg 1, B200 mode after the collective Step-1 calibration) over the
    direct NVLink path, the relays GPU2..GPU{N-1} and the pinned-host PCIe path (P:352's
    2_GPUs / 3_GPUs / 3_GPUs_w_host setups grown to N GPUs).  "scaling": "strong" — the
    message is fixed and N adds relay GPUs.  value = payload GB/s GPU0 → GPU1 over K
    back-to-back messages, max-over-ranks device time.  Baselines on the same pair:
    NCCL send/recv (before mp_init) and a copy-engine peer copy (cudaMemcpyAsync into
    the IPC-mapped receive buffer — what cudaMemcpyPeerAsync does).  Bootstrap and
    reductions use gloo on the CPU."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp

    dist.init_process_group("gloo")
    dev = rank_device(local, world)
    torch.cuda.set_device(dev)
    n = args.size
    roles = p2p_roles(world)
    role = roles[rank]
    s_tx, s_rx = torch.cuda.Stream(), torch.cuda.Stream()
    src = expect = None
    if role == "sender":
        src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                            generator=torch.Generator(device="cuda").manual_seed(20251116))
    if role == "receiver":
        expect = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                               generator=torch.Generator(device="cuda").manual_seed(20251116))
    torch.cuda.synchronize()
    base = {}

    # NCCL send/recv on the same pair (context, not the product), before mp_init
    try:
        g_nccl = dist.new_group(backend="nccl")
        buf = src if role == "sender" else torch.empty(n, dtype=torch.uint8, device="cuda")
        nb_steps = max(3, min(args.steps, 20))
        tb = 0.0
        for it in range(nb_steps + 2):
            if it == 2:
                torch.cuda.synchronize()
                b0 = time.perf_counter()
            if role == "sender":
                dist.send(buf, 1, group=g_nccl)
            elif role == "receiver":
                dist.recv(buf, 0, group=g_nccl)
        torch.cuda.synchronize()
        tb = time.perf_counter() - b0 if role in ("sender", "receiver") else 0.0
        tb = _gather_max(tb)
        base["nccl_send_recv_GBps"] = n * nb_steps / tb / 1e9
        dist.destroy_process_group(g_nccl)
        del buf
        torch.cuda.synchronize()
    except Exception as exc:
        base["nccl_error"] = repr(exc)

    # Step 2: a parameter file of this topology replaces Step 1's calibration
    ctx = mdist.context_from_dist(device=dev, calibrate=not (args.no_calibrate or args.params),
                                  heap_bytes=n + 64 * MiB, timeout_s=60.0, param_file=args.params)
    if args.save_params and rank == 0:
        ctx.save_params(args.save_params)
    _, cfg = p2p_plan(ctx, world, n, args.mode)
    d = cfg.as_dict()
    topo = ctx.topology()
    _, prm01, port01 = ctx.get_model(0, 1)
    rbuf = ctx.alloc(n) if role == "receiver" else None
    rview = mp.as_tensor(rbuf, n) if rbuf else None

    def message(c, tag):
        if role == "sender":
            ctx.send(src, n, 1, tag, c, s_tx)
        elif role == "receiver":
            ctx.recv(rbuf, n, 0, tag, s_rx)

    def timed(c, k, tag0=0):
        """k messages with config c: max-over-ranks device time (s) between two events
        on each endpoint's stream, after a barrier."""
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        st = s_tx if role == "sender" else s_rx
        e0.record(st)
        for i in range(k):
            message(c, tag0 + i)
        e1.record(st)
        st.synchronize()
        ms = e0.elapsed_time(e1) if role in ("sender", "receiver") else 0.0
        return _gather_max(ms) * 1e-3

    for i in range(args.warmup):
        message(cfg, i)
    s_tx.synchronize()
    s_rx.synchronize()
    ctx.sync()
    if role == "receiver":
        assert torch.equal(rview, expect), "payload mismatch"
    dist.barrier()
    l0 = ctx.launches()
    with Clocks(dev) as clk:
        t = timed(cfg, args.steps)
    launches = int(_gather_sum(ctx.launches() - l0))
    ctx.sync()
    if role == "receiver":
        assert torch.equal(rview, expect), "payload mismatch (timed)"
    value = n * args.steps / t / 1e9

    # end to end through the public API: the sender's payload comes from pinned host
    # memory every step (H2D on its stream), the receiver reads every message back
    h_src = src.cpu().pin_memory() if role == "sender" else None
    h_dst = torch.empty(n, dtype=torch.uint8).pin_memory() if role == "receiver" else None
    e2e_steps = max(3, min(10, args.steps // 4))
    dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    st = s_tx if role == "sender" else s_rx
    e0.record(st)
    for i in range(e2e_steps):
        if role == "sender":
            with torch.cuda.stream(s_tx):
                src.copy_(h_src, non_blocking=True)
        message(cfg, 1000 + i)
        if role == "receiver":
            with torch.cuda.stream(s_rx):
                h_dst.copy_(rview, non_blocking=True)
    e1.record(st)
    st.synchronize()
    te = _gather_max(e0.elapsed_time(e1) if role in ("sender", "receiver") else 0.0) * 1e-3
    e2e = n * e2e_steps / te / 1e9
    if role == "receiver":
        assert torch.equal(h_dst, expect.cpu()), "payload mismatch (e2e)"

    # every path alone (A7-A9 evidence), a few messages each, same pair
    per_path = {}
    paths_ = d["paths"]
    kp = max(3, min(args.steps, 10))
    _, prm, _ = ctx.get_model(0, 1)
    for i, (kind, via) in enumerate(paths_):
        nb = [0] * len(paths_)
        nb[i] = n
        ks = [1] + [0] * (len(paths_) - 1)
        if i:
            ks[i] = max(16, -(-n // (32 * MiB - 512)))
        ti = timed(ctx.make_config(nb, ks, 0, 1), kp, 5000 + 100 * i)
        gbs = n / (ti / kp) / 1e9
        name = "direct" if kind == 0 else (f"relay_gpu{via}" if kind == 1 else "host_pcie")
        row = {"GBps": gbs, "chunks": ks[i]}
        if kind == 0:
            row.update({"frac_of_nvlink_nominal": gbs / 900.0, "frac_of_measured_peer_copy": gbs / 770.0})
        else:
            ceil = min(prm[i]["beta"], prm[i]["beta2"]) / 1e9
            row.update({"stage_group_ceiling_GBps": ceil, "frac_of_stage_group_ceiling": gbs / ceil})
            if kind == 2:
                row["frac_of_pcie_nominal"] = gbs / 64.0
        per_path[name] = row
    if role == "receiver":
        assert torch.equal(rview, expect), "payload mismatch (per-path)"

    # copy-engine peer copy GPU0 -> GPU1's receive buffer (what cudaMemcpyPeerAsync does)
    try:
        from cuda.bindings import runtime as rt
        offs = [None] * world
        dist.all_gather_object(offs, (rbuf - ctx.peer_base(rank)) if rbuf else None)
        ce_t = 0.0
        nb_steps = max(3, min(args.steps, 20))
        dist.barrier()
        if role == "sender":
            dptr = ctx.peer_base(1) + offs[1]
            kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for _ in range(2):
                rt.cudaMemcpyAsync(dptr, src.data_ptr(), n, kind, s_tx.cuda_stream)
            c0.record(s_tx)
            for _ in range(nb_steps):
                rt.cudaMemcpyAsync(dptr, src.data_ptr(), n, kind, s_tx.cuda_stream)
            c1.record(s_tx)
            s_tx.synchronize()
            ce_t = c0.elapsed_time(c1) * 1e-3 / nb_steps
        ce_t = _gather_max(ce_t)
        base["cudaMemcpyPeer_ce_GBps"] = n / ce_t / 1e9
        base["mp_over_cudaMemcpyPeer"] = value / base["cudaMemcpyPeer_ce_GBps"]
    except Exception as exc:
        base["peer_copy_error"] = repr(exc)
    if "nccl_send_recv_GBps" in base:
        base["mp_over_nccl"] = value / base["nccl_send_recv_GBps"]

    nvl = sum(b for (k, _), b in zip(paths_, d["bytes"]) if k != 2)
    host = n - nvl
    per_s = args.steps / t
    nvl_gbs, pcie_gbs = nvl * per_s / 1e9, host * per_s / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_nvlink.json")
    if os.path.exists(tp):  # scripts/ncu_rank.sh + scripts/nvlink_summary.py
        try:
            traffic = json.load(open(tp))[f"{world}:{n}"]["rank0:send_kernel"]["nvlink_tx_bytes_per_launch"]
        except Exception:
            traffic = None
    roofline = {"bound": "nvlink+pcie", "achieved": value, "peak": 964.0, "unit": "GB/s",
                "frac": value / 964.0, "traffic": traffic,
                "peak_source": "nominal summed path roofline of the source GPU: NVLink 5 egress 900 GB/s "
                               "+ PCIe Gen5 x16 64 GB/s (north star); measured peer copy 770 GB/s "
                               "(B200_PROFILING.md) alongside",
                "nvlink_egress_GBps": nvl_gbs, "frac_of_nvlink_nominal": nvl_gbs / 900.0,
                "frac_of_measured_peer_copy": nvl_gbs / 770.0, "pcie_GBps": pcie_gbs,
                "frac_of_pcie_nominal": pcie_gbs / 64.0, "kernel": "send_kernel + relay_kernel + recv_kernel"}
    clk_all = [None] * world
    dist.all_gather_object(clk_all, clk.summary())
    pred = n / d["t_pred"] / 1e9 if d["t_pred"] else None
    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t / args.steps * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8",
        "data": "synthetic (seeded uniform random bytes)", "config": workload_config(args, world, d),
        "roofline": roofline,
        "e2e": {"value": e2e, "unit": "GB/s", "h2d_bytes_per_step": n, "d2h_bytes_per_step": n},
        "gpu_launches": launches,
        "clocks": clk_all[0], "clocks_all_ranks": clk_all,
        "baselines": base, "per_path": per_path,
        "model": {"selected": d, "split": split_label(d), "predicted_GBps": pred,
                  "E_pred": abs(pred - value) / value if pred else None, "params": prm01, "port": port01},
        "topology": {"fingerprint": topo["fingerprint"],
                     "gpus": [{k: g[k] for k in ("numa_node", "pcie_gen", "pcie_width", "nvlinks", "sms")}
                              for g in topo["gpus"]],
                     "peer_access_all": all(all(r) for r in topo["peer_access"])},
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if rbuf:
        ctx.free(rbuf)
    ctx.close()
    dist.destroy_process_group()
    return 0


def run_world_pairs(args, world, rank, local):
    """N > 1 with --workload config5 (secondary line): BASELINE.json config 5, SURVEY §8(d)'s
    primary reading — disjoint pairs (0↔1, 2↔3, …) exchange one message each way per
    step, all pairs at once, so every GPU's NVLink egress and ingress are busy and
    every would-be relay is itself an endpoint.  Messages go through the multi-rank
    engine (IPC-mapped heaps, direct NVLink path, relays through the other GPUs,
    pinned-host PCIe path), model-selected after a collective calibration.
    value = bytes moved by all ranks / max-over-ranks time.  Bootstrap and the
    reductions use gloo on CPU: no NCCL kernel ever runs beside the relay kernel."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp

    dist.init_process_group("gloo")
    dev = rank_device(local, world)
    torch.cuda.set_device(dev)
    n = args.size
    peer = rank + 1 if rank % 2 == 0 else rank - 1
    active = peer < world
    npairs = world // 2
    # Initialise every CUDA kernel this process will use BEFORE mp_init.
    s_tx, s_rx = torch.cuda.Stream(), torch.cuda.Stream()
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                        generator=torch.Generator(device="cuda").manual_seed(20251116 + rank))
    expect = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                           generator=torch.Generator(device="cuda").manual_seed(20251116 + peer))
    h_src = torch.empty(n, dtype=torch.uint8).pin_memory()
    h_dst = torch.empty(n, dtype=torch.uint8).pin_memory()
    h_src.copy_(src)
    assert torch.equal(src, src.clone())
    torch.cuda.synchronize()

    # Baseline (context, not the product): NCCL send/recv between the same pairs, both
    # directions, measured before mp_init so no NCCL kernel runs beside the relay.
    base = {}
    if active:
        try:
            g_nccl = dist.new_group(backend="nccl")
            scratch = torch.empty_like(src)
            nb_steps = max(3, min(args.steps, 20))
            for it in range(nb_steps + 2):
                if it == 2:
                    torch.cuda.synchronize()
                    b0 = time.perf_counter()
                ops = [dist.P2POp(dist.isend, src, peer, g_nccl), dist.P2POp(dist.irecv, scratch, peer, g_nccl)]
                for w in dist.batch_isend_irecv(ops):
                    w.wait()
            torch.cuda.synchronize()
            tb = time.perf_counter() - b0
            base["nccl_send_recv_GBps_per_direction"] = n * nb_steps / tb / 1e9
            dist.destroy_process_group(g_nccl)
            del scratch
            torch.cuda.synchronize()
        except Exception as exc:
            base["nccl_error"] = repr(exc)

    ctx = mdist.context_from_dist(device=dev, calibrate=not (args.no_calibrate or args.params),
                                  heap_bytes=n + 64 * MiB, timeout_s=60.0, param_file=args.params)
    ctx.set_options(mode=mp.MP_MODEL_B200 if args.mode == "b200" else mp.MP_MODEL_PAPER)
    # the communication pattern is known ahead of time: select jointly for all
    # concurrent flows (NEXT f1, mp_select_flows) — every rank computes the same configs
    flows = [(r, r ^ 1, n, 0) for r in range(world) if (r ^ 1) < world]
    cfgs = ctx.select_flows(flows)
    my_cfg = cfgs[[f[0] for f in flows].index(rank)] if active else None
    d = (my_cfg or cfgs[0]).as_dict()
    rbuf = ctx.alloc(n) if active else None
    rview = mp.as_tensor(rbuf, n) if rbuf else None

    def step():
        if active:
            ctx.recv(rbuf, n, peer, 0, s_rx)
            ctx.send(src, n, peer, 0, my_cfg, s_tx)

    for _ in range(args.warmup):
        step()
    s_tx.synchronize()
    s_rx.synchronize()
    ctx.sync()
    if active:
        assert torch.equal(rview, expect), "payload mismatch"
    dist.barrier()
    l0 = ctx.launches()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    with Clocks(dev) as clk:
        t0.record(s_tx)
        s_rx.wait_event(t0)
        for _ in range(args.steps):
            step()
        s_tx.wait_stream(s_rx)
        t1.record(s_tx)
        s_tx.synchronize()
    ms = t0.elapsed_time(t1) if active else 0.0
    stats = torch.tensor([ms, float(ctx.launches() - l0)], dtype=torch.float64)
    mx = stats.clone()
    dist.all_reduce(mx, op=dist.ReduceOp.MAX)
    sm = stats.clone()
    dist.all_reduce(sm, op=dist.ReduceOp.SUM)
    ms = float(mx[0])
    value = 2 * n * npairs * args.steps / (ms * 1e-3) / 1e9

    # end to end: every step each sender's payload comes from pinned host memory and
    # each receiver reads its message back to pinned host memory.
    e2e_steps = max(3, min(10, args.steps // 4))
    dist.barrier()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s_tx)
    s_rx.wait_event(e0)
    for _ in range(e2e_steps):
        if active:
            with torch.cuda.stream(s_tx):
                src.copy_(h_src, non_blocking=True)
        step()
        if active:
            with torch.cuda.stream(s_rx):
                h_dst.copy_(rview, non_blocking=True)
    s_tx.wait_stream(s_rx)
    e1.record(s_tx)
    s_tx.synchronize()
    e = torch.tensor([e0.elapsed_time(e1) if active else 0.0], dtype=torch.float64)
    dist.all_reduce(e, op=dist.ReduceOp.MAX)
    e2e = 2 * n * npairs * e2e_steps / (float(e[0]) * 1e-3) / 1e9

    # Baseline: the single-path copy-engine peer copy (what cudaMemcpyPeerAsync does),
    # both directions at once, through the IPC mapping of the partner's heap buffer.
    try:
        from cuda.bindings import runtime as rt
        offs = [None] * world
        dist.all_gather_object(offs, (rbuf - ctx.peer_base(rank)) if rbuf else None)
        ce_t = 0.0
        if active:
            dptr = ctx.peer_base(peer) + offs[peer]
            kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
            c0 = torch.cuda.Event(enable_timing=True)
            c1 = torch.cuda.Event(enable_timing=True)
            dist.barrier()
            for _ in range(2):
                rt.cudaMemcpyAsync(dptr, src.data_ptr(), n, kind, s_tx.cuda_stream)
            c0.record(s_tx)
            nb_steps = max(3, min(args.steps, 20))
            for _ in range(nb_steps):
                rt.cudaMemcpyAsync(dptr, src.data_ptr(), n, kind, s_tx.cuda_stream)
            c1.record(s_tx)
            s_tx.synchronize()
            ce_t = c0.elapsed_time(c1) * 1e-3 / nb_steps
        else:
            dist.barrier()
        tt = torch.tensor([ce_t], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        base["cudaMemcpy_peer_GBps_per_direction"] = n / float(tt[0]) / 1e9
    except Exception as exc:
        base["peer_copy_error"] = repr(exc)

    nvl = sum(b for (k, _), b in zip(d["paths"], d["bytes"]) if k != 2)
    per_dir = n * args.steps / (ms * 1e-3) / 1e9
    achieved = nvl * args.steps / (ms * 1e-3) / 1e9
    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic (seeded uniform random bytes)",
        "config": workload_config(args, world, d),
        "roofline": ({"bound": "nvlink", "achieved": achieved, "peak": 770.0, "unit": "GB/s",
                      "frac": achieved / 770.0, "traffic": None, "peak_source":
                      "B200_PROFILING.md measured peer copy, per direction per GPU (nominal 900)",
                      "kernel": "send_kernel"}),
        "per_direction_GBps": per_dir,
        "baselines": base,
        "e2e": {"value": e2e, "unit": "GB/s", "h2d_bytes_per_step": n * 2 * npairs,
                "d2h_bytes_per_step": n * 2 * npairs},
        "gpu_launches": int(sm[1]),
        "clocks": clk.summary(),
        "model": {"selected": d, "predicted_GBps": n / d["t_pred"] / 1e9 if d["t_pred"] else None,
                  "E_pred": abs(n / d["t_pred"] / 1e9 - per_dir) / per_dir if d["t_pred"] else None},
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if rbuf:
        ctx.free(rbuf)
    ctx.close()
    dist.destroy_process_group()
    return 0


def selector_overhead(ctx, n, gbps):
    """E5 (the model's runtime overhead, "<0.1 % of the total execution
    time" for large messages): mp_select per call through the binding, on a cache
    miss (every call a new size) and a hit, against the message's measured time."""
    k = 2000
    t0 = time.perf_counter()
    for i in range(k):
        ctx.select(0, 0, n + 256 * (i + 1))
    miss = (time.perf_counter() - t0) / k
    t0 = time.perf_counter()
    for _ in range(k):
        ctx.select(0, 0, n)
    hit = (time.perf_counter() - t0) / k
    t_msg = n / (gbps * 1e9)
    return {"miss_us": miss * 1e6, "hit_us": hit * 1e6, "miss_frac_of_message": miss / t_msg,
            "note": "Python ctypes call included; the message is the timed 1 GiB transfer"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="mpx", choices=["mpx", "reference"])
    ap.add_argument("--size", type=int, default=None,
                    help="message bytes (default: 1 GiB — config 3; 256 MiB per message with --workload config5)")
    ap.add_argument("--mode", default="b200", choices=["b200", "paper"])
    ap.add_argument("--workload", default="config3", choices=["config3", "config5"],
                    help="N > 1: config3 (GPU0 -> GPU1 over direct + relays GPU2.. + host; default) or "
                         "config5 (disjoint pairs exchanging, every GPU busy)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-calibrate", action="store_true",
                    help="skip the init-time calibration (default parameters; for ncu runs)")
    ap.add_argument("--params", default=None, help="load model parameters (Step 2) instead of calibrating")
    ap.add_argument("--save-params", default=None, help="write the calibrated parameters (Step 1)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.size is None:
        args.size = 256 * MiB if (args.workload == "config5" and int(os.environ.get("WORLD_SIZE", "1")) > 1) else GiB
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_sojoodiasfga25_b200 import mp

    world, rank, local = dist_env()
    if world > 1:
        return run_world(args, world, rank, local)
    torch.cuda.set_device(local)
    n = args.size
    ctx = mp.Context(device=local, calibrate=not (args.no_calibrate or args.params), n_loop_relays=6,
                     host_path=1, heap_bytes=16 * MiB, param_file=args.params)
    if args.save_params and rank == 0:
        ctx.save_params(args.save_params)
    ctx.set_options(mode=mp.MP_MODEL_B200 if args.mode == "b200" else mp.MP_MODEL_PAPER)
    cfg = ctx.select(0, 0, n)
    d = cfg.as_dict()
    stream = torch.cuda.Stream()
    g = torch.Generator(device="cuda").manual_seed(20251116 + rank)
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda", generator=g)
    dst = torch.empty(n, dtype=torch.uint8, device="cuda")

    def step():
        ctx.xfer(dst, src, n, None, stream)   # mp_select (cached) + one fused launch

    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            step()
    torch.cuda.synchronize()
    ctx.sync()
    assert torch.equal(dst, src), "payload mismatch"

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = ctx.launches()
    # The timed region: K back-to-back steps between two events on the launching
    # stream.  Each step is one kernel launch (gpu_launches), so (t1 − t0)/K is the
    # kernel's average launch duration; consecutive launches overlap their launch
    # latency by PDL, which an event record between them would undo.
    with Clocks(local) as clk:
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for i in range(args.steps):
            step()
        t1.record(stream)
        torch.cuda.synchronize()
    launches = ctx.launches() - l0
    ctx.sync()
    ms = t0.elapsed_time(t1)
    # per-launch spread: a separate pass with events around every launch (each event
    # record also costs ~2.5 µs of stream time, so these are upper bounds)
    nev = min(args.steps, 200)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nev)]
    for i in range(nev):
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    per_launch = sorted(a.elapsed_time(b) for a, b in ev)
    ms_t = torch.tensor([ms], device="cuda")
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
        dist.barrier()
    ms = float(ms_t.item())
    value = n * world * args.steps / (ms * 1e-3) / 1e9

    # end to end through the public API with host buffers: every step copies its
    # payload host→device from pinned memory, runs the transfer, and reads the received
    # message back device→host.  Steps are software-pipelined over two buffer sets and
    # three streams so the H2D of step i+1 overlaps the D2H of step i (PCIe is full
    # duplex); every byte still crosses PCIe both ways inside the timed region.
    h_src = src.cpu().pin_memory()
    h_dst = [torch.empty(n, dtype=torch.uint8).pin_memory() for _ in range(2)]
    srcs = [src, torch.empty_like(src)]
    dsts = [dst, torch.empty_like(dst)]
    s_up, s_dn = torch.cuda.Stream(), torch.cuda.Stream()
    # enough steps that the pipeline's fill (the first H2D and the last D2H, which
    # overlap nothing) is a small part of the timed region
    e2e_steps = max(3, min(48, args.steps // 4))
    torch.cuda.synchronize()
    ev = lambda: torch.cuda.Event()  # noqa: E731
    up_done, x_done, dn_done = [ev(), ev()], [ev(), ev()], [ev(), ev()]
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    s_up.wait_event(e0)
    for i in range(e2e_steps):
        b = i % 2
        if i >= 2:
            s_up.wait_event(x_done[b])            # srcs[b] free (step i-2 read it)
        with torch.cuda.stream(s_up):
            srcs[b].copy_(h_src, non_blocking=True)
        up_done[b].record(s_up)
        stream.wait_event(up_done[b])
        if i >= 2:
            stream.wait_event(dn_done[b])         # dsts[b] free (step i-2 read back)
        ctx.xfer(dsts[b], srcs[b], n, None, stream)
        x_done[b].record(stream)
        s_dn.wait_event(x_done[b])
        with torch.cuda.stream(s_dn):
            h_dst[b].copy_(dsts[b], non_blocking=True)
        dn_done[b].record(s_dn)
    stream.wait_event(dn_done[(e2e_steps - 1) % 2])
    stream.wait_event(dn_done[(e2e_steps - 2) % 2])
    e1.record(stream)
    torch.cuda.synchronize()
    e2e = n * e2e_steps / (e0.elapsed_time(e1) * 1e-3) / 1e9
    assert torch.equal(h_dst[0], h_src) and torch.equal(h_dst[1], h_src)

    # Per-row evidence for the staged legs (§8(a) A8, A9), which the B200-mode pick
    # leaves idle on this topology: each staged path alone, and the paper-mode pick
    # (every path carrying bytes), each the median of 5 fused launches.
    def med(fn, reps=5):
        ts = []
        for _ in range(reps + 1):
            a0 = torch.cuda.Event(enable_timing=True)
            a1 = torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            fn()
            a1.record(stream)
            a1.synchronize()
            ts.append(a0.elapsed_time(a1) * 1e-3)
        ts = sorted(ts[1:])
        return ts[len(ts) // 2]

    per_path = {}
    peak, peak_src = measured_peaks()
    paths_ = d["paths"]
    nstage = 256 * MiB
    for name, idx in (("relay_ring_alone", 1), ("host_pcie_alone", len(paths_) - 1)):
        nb = [0] * len(paths_)
        nb[idx] = nstage
        ks = [1] + [0] * (len(paths_) - 1)
        ks[idx] = 16
        cfg_s = ctx.make_config(nb, ks)
        t = med(lambda: ctx.xfer(dst, src, nstage, cfg_s, stream))
        gbs = nstage / t / 1e9
        if name.startswith("relay"):
            # a staged path is two stage groups of relay_ctas (16) CTAs each, sized for
            # a relay's NVLink share beside the direct group, not for loopback HBM: its
            # ceiling is the slower leg as Step 1 measured it with that group
            # (calibrated β, β' of the path)
            lp = ctx.get_model(0, 0)[1][idx]
            ceil_ = min(lp["beta"], lp["beta2"]) / 1e9
            per_path[name] = {"GBps": gbs, "bytes": nstage, "chunks": 16, "bound": "hbm",
                              "hbm_GBps": 4 * nstage / t / 1e9, "frac": 4 * nstage / t / 1e9 / peak,
                              "ctas": 32, "hbm_GBps_per_cta": 4 * nstage / t / 1e9 / 32,
                              "stage_group_ceiling_GBps": ceil_, "frac_of_stage_group_ceiling": gbs / ceil_}
        else:
            per_path[name] = {"GBps": gbs, "bytes": nstage, "chunks": 16, "bound": "pcie",
                              "peak": 64.0, "frac": gbs / 64.0,
                              "peak_source": "PCIe Gen5 x16 nominal per direction (north star)"}
    # the practical ceiling of SM-driven PCIe traffic in loopback: both host legs share
    # this GPU's link, so a full-grid SM copy device→pinned host and one pinned
    # host→device, run at once, bound what the host path can reach
    try:
        hp = torch.empty(nstage, dtype=torch.uint8).pin_memory()
        hq = torch.empty(nstage, dtype=torch.uint8).pin_memory()
        s2 = torch.cuda.Stream()
        dcfg = ctx.make_config([nstage] + [0] * (len(paths_) - 1), [1] + [0] * (len(paths_) - 1))

        def duplex():
            e = torch.cuda.Event()
            e.record(stream)
            s2.wait_event(e)
            ctx.xfer(hp.data_ptr(), src, nstage, dcfg, stream)
            ctx.xfer(dst, hq.data_ptr(), nstage, dcfg, s2)
            e2 = torch.cuda.Event()
            e2.record(s2)
            stream.wait_event(e2)
        ceil = nstage / med(duplex) / 1e9
        h = per_path["host_pcie_alone"]
        h["sm_duplex_ceiling_GBps"] = ceil
        h["frac_of_sm_duplex_ceiling"] = h["GBps"] / ceil
        del hp, hq
    except Exception as exc:  # context, not the product
        per_path["host_pcie_alone"]["sm_duplex_ceiling_error"] = repr(exc)
    ctx.set_options(mode=mp.MP_MODEL_PAPER)
    pcfg = ctx.select(0, 0, n)
    t = med(lambda: ctx.xfer(dst, src, n, pcfg, stream))
    pd = pcfg.as_dict()
    per_path["paper_mode_pick_all_paths"] = {"GBps": n / t / 1e9, "bytes": pd["bytes"], "chunks": pd["chunks"],
                                             "split": split_label(pd), "kernel": "xfer_kernel",
                                             "hbm_GBps": hbm_bytes(pd) / t / 1e9,
                                             "frac": hbm_bytes(pd) / t / 1e9 / peak,
                                             "vs_b200_pick": (n / t / 1e9) / (value / world)}
    ctx.set_options(mode=mp.MP_MODEL_B200 if args.mode == "b200" else mp.MP_MODEL_PAPER)

    # The metric's second half, "model-vs-sweep optimum error %" (a static
    # exhaustive-search split against the model's dynamic one): a compact sweep at this
    # message size — direct alone; direct + host; direct + 1 or all relays, ± host; k in
    # {1, 4} — each config the median of 5 windows of 2 back-to-back launches behind a
    # spin kernel, the model's pick timed the same way (scripts/sweep.py runs the full
    # grid at 16 MiB - 1 GiB: profiles/r02/sweep_summary*.jsonl).
    def window(cfg_w, W=2, reps=5):
        ts = []
        for r in range(reps + 1):
            w0 = torch.cuda.Event(enable_timing=True)
            w1 = torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(stream):
                torch.cuda._sleep(2_000_000)
            w0.record(stream)
            for _ in range(W):
                ctx.xfer(dst, src, n, cfg_w, stream)
            w1.record(stream)
            w1.synchronize()
            if r:
                ts.append(w0.elapsed_time(w1) * 1e-3 / W)
        ts.sort()
        return ts[len(ts) // 2]

    e_sel = None
    try:
        rows = []
        for nb, ch in esel_grid(n, len(paths_), len(paths_) - 1):
            rows.append({"bytes": nb, "chunks": ch, "GBps": n / window(ctx.make_config(nb, ch)) / 1e9})
        best = max(rows, key=lambda r: r["GBps"])
        pick_gbs = n / window(ctx.make_config(d["bytes"], d["chunks"])) / 1e9
        pred = n / d["t_pred"] / 1e9 if d["t_pred"] else None
        e_sel = {"value": 100.0 * max(0.0, 1 - pick_gbs / best["GBps"]), "unit": "%", "n_configs": len(rows),
                 "pick_GBps": pick_gbs, "pick_split": split_label(d), "best_GBps": best["GBps"],
                 "best_split": split_label({"paths": paths_, "bytes": best["bytes"], "chunks": best["chunks"]}),
                 "E_pred_vs_best_pct": 100.0 * abs(pred - best["GBps"]) / best["GBps"] if pred else None,
                 "method": "windows of 2 back-to-back launches behind a spin kernel, median of 5"}
    except Exception as exc:  # context; the product number is `value`
        e_sel = {"error": repr(exc)}
    torch.cuda.synchronize()
    assert torch.equal(dst, src), "payload mismatch (per-path runs)"

    # single-path baseline: cudaMemcpyAsync device→device on the same stream (the
    # copy the paper's engine issues per chunk), same buffers and timing.
    base = None
    try:
        from cuda.bindings import runtime as rt
        kind = rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice
        bsteps = max(5, min(args.steps, 50))
        b0 = torch.cuda.Event(enable_timing=True)
        b1 = torch.cuda.Event(enable_timing=True)
        for _ in range(3):
            rt.cudaMemcpyAsync(dst.data_ptr(), src.data_ptr(), n, kind, stream.cuda_stream)
        b0.record(stream)
        for _ in range(bsteps):
            rt.cudaMemcpyAsync(dst.data_ptr(), src.data_ptr(), n, kind, stream.cuda_stream)
        b1.record(stream)
        torch.cuda.synchronize()
        base = {"cudaMemcpyAsync_d2d_GBps": n * bsteps / (b0.elapsed_time(b1) * 1e-3) / 1e9,
                "steps": bsteps}
    except Exception as exc:  # the baseline is context, not the product
        base = {"error": repr(exc)}

    # The multi-rank kernels on this one GPU: config 3's message size from
    # rank 0 to rank 1 of an emulated world of 3 (direct + relay rank 2 + host), every
    # rank's kernels in one cooperative grid; checked on the device against the source.
    # One GPU: every path is an HBM copy, so this is the kernels' rate, not NVLink's.
    emu = None
    try:
        torch.cuda.synchronize()
        with mp.EmulatedWorld(3, device=0, heap_bytes=n + 64 * MiB, timeout_s=60.0) as W:
            e0c, e1c = W.ctx[0], W.ctx[1]
            rb, hb = n // 8 // 256 * 256, n // 512 // 256 * 256  # ~ the paper-mode pick's relay / host shares
            enb = [n - rb - hb, rb, hb]
            eks = [1, max(1, rb // (16 * MiB)), max(1, hb // (16 * MiB))]
            ecfg = e0c.make_config(enb, eks, 0, 1)
            edst = e1c.alloc(n)
            eview = mp.as_tensor(edst, n)
            ts = []
            for r in range(4):
                e0c.send(src, n, 1, tag=r, cfg=ecfg)
                e1c.recv(edst, n, 0, tag=r)
                ts.append(W.run(stream))
            ok = bool(torch.equal(eview, src))
            t = sorted(ts[1:])[1]
            emu = {"world": 3, "msg_bytes": n, "split": split_label({"paths": e0c.paths(0, 1), "bytes": enb,
                                                                      "chunks": eks}),
                   "GBps": n / t / 1e9, "grid_ms": t * 1e3, "bit_exact": ok,
                   "hbm_GBps": (2 * enb[0] + 4 * enb[1] + 2 * enb[2]) / t / 1e9,
                   "hbm_frac": (2 * enb[0] + 4 * enb[1] + 2 * enb[2]) / t / 1e9 / measured_peaks()[0],
                   "kernel": "emu_kernel: send gate, send, relay and receive bodies in one cooperative grid",
                   "note": "one GPU: HBM copies, not NVLink; timing = CUDA events around the grid"}
            e1c.free(edst)
            del eview
    except Exception as exc:  # evidence for the multi-rank kernels, not the product number
        emu = {"error": repr(exc)}

    peak, peak_src = measured_peaks()
    alg = hbm_bytes(d)
    avg_launch_ms = ms / args.steps  # the timed region's average launch duration
    achieved = alg / (avg_launch_ms * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(str(n), {}).get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    _, prm, port = ctx.get_model(0, 0)
    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic (seeded uniform random bytes)",
        "config": workload_config(args, world, d),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "peak_source": peak_src,
                     "kernel": "direct_kernel" if all(b == 0 for b in d["bytes"][1:]) else "xfer_kernel",
                     "algorithmic_bytes_per_launch": alg,
                     "note": "achieved = algorithmic bytes / (timed region / steps); the peak is "
                             "torch copy_ timed alone, this kernel runs back to back under PDL"},
        "e2e": {"value": e2e, "unit": "GB/s", "h2d_bytes_per_step": n, "d2h_bytes_per_step": n},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "model": {"selected": d, "predicted_GBps": n / d["t_pred"] / 1e9 if d["t_pred"] else None,
                  "E_pred": abs(n / d["t_pred"] / 1e9 - value / world) / (value / world) if d["t_pred"] else None,
                  "port": port, "direct_params": prm[0], "host_params": prm[-1]},
        "per_launch_ms": {"timed_region_avg": avg_launch_ms, "evented_pass_launches": len(per_launch),
                          "min": per_launch[0], "median": per_launch[len(per_launch) // 2],
                          "max": per_launch[-1]},
        "baselines": base,
        "e_sel": e_sel,
        "emulated_multirank": emu,
        "per_path": per_path,
        "select_overhead": selector_overhead(ctx, n, value / world),
        "topology": {k: v for k, v in ctx.topology().items() if k in ("fingerprint", "gpus")},
    }
    # NEXT f4 (readings C20/C21): the same message modelled with per-band Step-1
    # parameters (calibrated after the timed region; the pick is unchanged at 1 GiB)
    if not (args.no_calibrate or args.params):
        try:
            ctx.calibrate_bands()
            bd = ctx.select(0, 0, n).as_dict()
            pb = n / bd["t_pred"] / 1e9
            line["model"]["bands"] = {"predicted_GBps": pb, "E_pred": abs(pb - value / world) / (value / world),
                                      "same_pick": bd["bytes"] == d["bytes"]}
        except Exception as exc:  # context, not the product
            line["model"]["bands"] = {"error": repr(exc)}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_oracle_run(n, d, prm)
    if rank == 0:
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
