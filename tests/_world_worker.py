"""Worker for the multi-rank tests (one process per rank, one GPU per rank: rank r on
device r — ranks whose kernels wait on one another never share a GPU; the one-GPU
stand-in is the emulated world, tests/test_emulated_gpu.py).

    python tests/_world_worker.py <rank> <world> <port> <scenario>

Scenario "gloo_model" (CPU): model-only contexts bootstrapped over gloo; every rank
selects the same configs and the all-gather callback round-trips.
Scenario "engine" (GPU): real multi-rank engine — IPC-mapped heaps, the on-demand
relay kernels, the shared pinned host ring — with rank 0 → rank 1 messages over every
path kind, checked byte for byte against the oracle reference transfer.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import ctypes  # noqa: E402

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

MiB = 1 << 20
DEV = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 0  # this rank's GPU


def scenario_gloo_model(rank, world):
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    ag = mdist.torch_allgather()
    inp = bytes([rank + 1] * 8)
    out = ctypes.create_string_buffer(8 * world)
    assert ag(None, inp, ctypes.addressof(out), 8) == 0
    assert out.raw == b"".join(bytes([r + 1] * 8) for r in range(world))
    c = mdist.context_from_dist(model_only=True)
    assert c.world == world and c.rank == rank
    cfgs = []
    for dst in range(world):
        if dst == rank:
            continue
        d = c.select(rank, dst, 256 * MiB).as_dict()
        assert sum(d["bytes"]) == 256 * MiB
        assert len(d["paths"]) == world  # direct + (world-2) relays + host
        cfgs.append((rank, dst, d["bytes"], d["chunks"]))
    # every rank computes the same selection for the same pair (pure function of the model)
    gathered = [None] * world
    dist.all_gather_object(gathered, c.select(0, 1, 64 * MiB).as_dict())
    assert all(g == gathered[0] for g in gathered)
    c.close()


def scenario_engine(rank, world):
    import numpy as np

    import synth
    from oracle import transfer as X
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    # Everything CUDA this process will need is initialised BEFORE mp_init: with
    # (round 1: a persistent relay kernel forbade an idle-device wait later; round 2's
    # relay kernels are bounded — scenario "devsync" — but this order is kept), and driver calls that
    # need an idle context (lazy module loading, torch's lazy init, first-use pools)
    # would wait for it forever.
    stream = torch.cuda.Stream()
    src_buf = torch.empty(8 * MiB, dtype=torch.uint8, device="cuda")
    src_buf.copy_(torch.from_numpy(synth.payload(8 * MiB, 0)))
    assert int(src_buf[:16].cpu().sum()) >= 0
    torch.cuda.synchronize()
    print(f"rank {rank}: init", flush=True)
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0)
    if world >= 3:
        # collective Step 1 after mp_init (the relay service keeps running)
        c.calibrate(sizes=[4 * MiB, 8 * MiB, 16 * MiB], reps=2)
        _, prm, _ = c.get_model(0, 1)
        assert prm[0]["beta"] > 0 and prm[1]["eps"] > 0
        # NEXT f2 (reading C25): every rank's host duplex factor is measured and shared
        assert all(0 < c.get_host_duplex(g) <= 1 for g in range(world))
    # NEXT f4: collective per-band Step 1 (readings C20/C21) on every pair
    c.calibrate_bands([0, 1 * MiB, 8 * MiB], reps=2)
    for dst in range(world):
        if dst == rank:
            continue
        bands = c.get_model_bands(rank, dst)
        assert [b[0] for b in bands] == [0, 1 * MiB, 8 * MiB], bands
        for _, prm, port in bands:
            assert all(p["beta"] > 0 and p["alpha"] > 0 for p in prm) and port["beta"] > 0
    ps = c.paths(0, 1)
    np_ = len(ps)
    cases = []
    n = 3 * MiB + 4099
    cases.append(([n] + [0] * (np_ - 1), [1] + [0] * (np_ - 1), n))                 # direct only
    relay_ok = os.environ.get("MPX_NO_RELAY") != "1"
    if world >= 3 and relay_ok:
        nb = [0] * np_
        nb[1] = n                                                               # one relay alone, k = 5
        ks = [1] + [0] * (np_ - 1)
        ks[1] = 5
        cases.append((nb, ks, n))
    nb = [0] * np_
    nb[-1] = n                                                                  # host path alone, k = 4
    ks = [1] + [0] * (np_ - 1)
    ks[-1] = 4
    cases.append((nb, ks, n))
    nb = [0] + [256 * 1024 if (relay_ok or k == 2) else 0 for k, _ in ps[1:]]      # every path at once
    nb[0] = n - sum(nb)
    cases.append((nb, [1] + [2 if b else 0 for b in nb[1:]], n))
    if relay_ok:
        cases.append((None, None, 5 * MiB + 1))                                 # model-selected
    else:
        d = c.select(0, 1, 5 * MiB + 1, 1 | (1 << (np_ - 1))).as_dict()
        cases.append((d["bytes"], d["chunks"], 5 * MiB + 1))
    print(f"rank {rank}: context up, {len(cases)} cases", flush=True)
    for i, (nb, ks, n) in enumerate(cases):
        print(f"rank {rank}: case {i} {nb} {ks}", flush=True)
        if rank == 0:
            host = synth.payload(n, i)
            src = src_buf[:n]
            src.copy_(torch.from_numpy(host))
            cfg = c.make_config(nb, ks, 0, 1) if nb else None
            c.send(src, n, 1, tag=100 + i, cfg=cfg, stream=stream)
            stream.synchronize()
        elif rank == 1:
            p = c.alloc(n)
            c.recv(p, n, 0, tag=100 + i, stream=stream)
            stream.synchronize()
            got = mp.as_tensor(p, n)
            host = synth.payload(n, i)
            exp = np.zeros(n, dtype=np.uint8)
            if nb:
                X.replay(host, nb, ks, [k for k, _ in ps], 256, exp)
            else:
                exp[:] = host
            assert np.array_equal(got.cpu().numpy(), exp), f"case {i} mismatch"
            c.free(p)
        dist.barrier()
    # a zero-byte message (allowed, moves nothing) completes and keeps
    # the pair's FIFO matching in step: the next message still arrives intact
    if rank == 0:
        src_buf[:4096].copy_(torch.from_numpy(synth.payload(4096, 77)))
        c.send(src_buf[:0], 0, 1, tag=90, stream=stream)
        c.send(src_buf[:4096], 4096, 1, tag=91, stream=stream)
        stream.synchronize()
    elif rank == 1:
        p = c.alloc(4096)
        c.recv(p, 0, 0, tag=90, stream=stream)
        c.recv(p, 4096, 0, tag=91, stream=stream)
        stream.synchronize()
        assert np.array_equal(mp.as_tensor(p, 4096).cpu().numpy(), synth.payload(4096, 77)), \
            "after a zero-byte message"
        c.free(p)
    dist.barrier()
    # bidirectional (osu_bibw-style): 0 → 1 and 1 → 0 at once, model-selected, two
    # streams per rank, a window of 3 messages each way
    if rank in (0, 1):
        other = 1 - rank
        s_tx, s_rx = torch.cuda.Stream(), torch.cuda.Stream()
        nbi = 2 * MiB + 77
        bufs = [c.alloc(nbi) for _ in range(3)]
        with torch.cuda.stream(s_tx):
            src_buf[:nbi].copy_(torch.from_numpy(synth.payload(nbi, 40 + rank)))
        for w in range(3):
            c.recv(bufs[w], nbi, other, tag=900 + w, stream=s_rx)
            c.send(src_buf[:nbi], nbi, other, tag=900 + w, stream=s_tx)
        s_tx.synchronize()
        s_rx.synchronize()
        exp = torch.from_numpy(synth.payload(nbi, 40 + other))
        for w in range(3):
            assert torch.equal(mp.as_tensor(bufs[w], nbi).cpu(), exp), f"bibw window {w}"
            c.free(bufs[w])
    dist.barrier()
    # the reverse direction alone
    if rank == 1:
        src = src_buf[:MiB]
        src.copy_(torch.from_numpy(synth.payload(MiB, 9)))
        c.send(src, MiB, 0, tag=5, stream=stream)
        stream.synchronize()
    elif rank == 0:
        p = c.alloc(MiB)
        c.recv(p, MiB, 1, tag=5, stream=stream)
        stream.synchronize()
        c.sync()
        c.free(p)
    dist.barrier()
    c.sync()
    assert c.launches() > 0 or rank >= 2
    c.close()


def scenario_faults(rank, world):
    """A tag mismatch is reported on both sides as MP_ERR_MISMATCH and a receive that
    is never matched ends in MP_ERR_TIMEOUT — on the device, bounded by %globaltimer —
    instead of hanging (failure detection)."""
    import synth
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    src = torch.empty(2 * MiB, dtype=torch.uint8, device="cuda")
    src.copy_(torch.from_numpy(synth.payload(2 * MiB, 0)))
    torch.cuda.synchronize()
    for fault in ("mismatch", "timeout", "eager_mismatch"):
        c = mdist.context_from_dist(device=DEV, heap_bytes=16 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                    timeout_s=3.0)
        nb = 4096 if fault == "eager_mismatch" else 2 * MiB   # 2 MiB: past the eager limit (rendezvous)
        if rank == 0 and fault != "timeout":
            c.send(src[:nb], nb, 1, tag=5, stream=stream)
        elif rank == 1:
            p = c.alloc(nb)
            c.recv(p, nb, 0, tag=7 if fault == "timeout" else 6, stream=stream)
        stream.synchronize()
        status = 0
        try:
            c.sync()
        except mp.MPError as e:
            status = e.status
        expect = {"mismatch": -8, "timeout": -7 if rank == 1 else 0,
                  "eager_mismatch": -8 if rank == 1 else 0}[fault]
        assert status == expect, (fault, rank, status)
        print(f"rank {rank}: {fault} -> {status}", flush=True)
        dist.barrier()
        c.close()


def scenario_register(rank, world):
    """mp_register (D7): receive into arbitrary torch tensors — two views of one
    torch allocation on rank 1 (a shared IPC mapping on every peer), then one tensor
    per rank in a ring — over every path at once, byte-exact against the oracle
    replay, bytes outside the views untouched; deregistered regions are refused."""
    import numpy as np

    import synth
    from oracle import transfer as X
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    big = torch.zeros(16 * MiB, dtype=torch.uint8, device="cuda")        # rank 1's targets
    ring = torch.zeros(4 * MiB, dtype=torch.uint8, device="cuda")        # every rank's ring target
    src_buf = torch.empty(8 * MiB, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=16 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0)
    ps = c.paths(0, 1)
    kinds = [k for k, _ in ps]
    va, vb = big[MiB + 256: 9 * MiB], big[10 * MiB: 15 * MiB]
    ida = c.register(va if rank == 1 else None)
    idb = c.register(vb if rank == 1 else None)
    idr = c.register(ring)
    assert len({ida, idb, idr}) == 3 and min(ida, idb, idr) >= 1
    # (region A) every path at once, explicit config; (region B) model-selected
    na = 3 * MiB + 4099
    nb = [256 * 1024] * len(ps)
    nb[0] = na - 256 * 1024 * (len(ps) - 1)
    ks = [1] + [2] * (len(ps) - 1)
    for case, (view, n, cfgb, cfgk) in enumerate([(va, na, nb, ks), (vb, 5 * MiB, None, None)]):
        host = synth.payload(n, 60 + case)
        if rank == 0:
            with torch.cuda.stream(stream):
                src_buf[:n].copy_(torch.from_numpy(host))
            c.send(src_buf[:n], n, 1, tag=300 + case, cfg=c.make_config(cfgb, cfgk, 0, 1) if cfgb else None,
                   stream=stream)
            stream.synchronize()
        elif rank == 1:
            c.recv(view[:n], n, 0, tag=300 + case, stream=stream)
            stream.synchronize()
            exp = host.copy()
            if cfgb:
                exp = np.zeros(n, dtype=np.uint8)
                X.replay(host, cfgb, cfgk, kinds, 256, exp)
            got = view[:n].cpu().numpy()
            bad = np.nonzero(got != exp)[0]
            assert bad.size == 0, (f"region case {case}: {bad.size} bytes differ, first {bad[:4]}, "
                                   f"last {bad[-4:]}, config {cfgb} {cfgk}")
        dist.barrier()
    # ring: rank r → r+1 into the peer's registered tensor, at a 4 KiB + 17 offset
    n = 2 * MiB + 333
    nxt, prv = (rank + 1) % world, (rank - 1) % world
    with torch.cuda.stream(stream):
        src_buf[:n].copy_(torch.from_numpy(synth.payload(n, 70 + rank)))
    s_rx = torch.cuda.Stream()
    c.recv(ring[4096 + 17: 4096 + 17 + n], n, prv, tag=400, stream=s_rx)
    c.send(src_buf[:n], n, nxt, tag=400, stream=stream)
    stream.synchronize()
    s_rx.synchronize()
    c.sync()
    assert np.array_equal(ring[4096 + 17: 4096 + 17 + n].cpu().numpy(), synth.payload(n, 70 + prv)), "ring"
    dist.barrier()
    for rid in (ida, idb, idr):
        c.deregister(rid)
    if rank == 1:
        try:
            c.recv(va[:MiB], MiB, 0, tag=1, stream=stream)
            raise AssertionError("recv into a deregistered region was accepted")
        except mp.MPError:
            pass
    # ids are reused after deregistration
    assert c.register(ring) == ida
    c.deregister(ida)
    dist.barrier()
    c.sync()
    c.close()
    # new torch kernels only now: a first launch lazily loads its module, which waits
    # for the device to idle
    if rank == 1:
        h = big.cpu().numpy()
        rest = np.concatenate([h[:MiB + 256], h[MiB + 256 + na: 10 * MiB], h[15 * MiB:]])
        assert not rest.any(), "bytes outside the registered views were written"


def scenario_eager(rank, world):
    """The eager protocol (reading C23): messages of 1 B..1 MiB, misaligned sources and
    destinations, 16-KiB slice edges, the 1 MiB / 1 MiB + 1 boundary to the rendezvous,
    a window of 20 messages (more than the 8 slots: flow control), and eager and
    rendezvous messages interleaved on one pair — every byte checked."""
    import numpy as np

    import synth
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    src_buf = torch.empty(3 * MiB, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0)
    sizes = [1, 17, 4095, 16384, 16385, 3 * 16384 + 5, 65537, 300000, MiB - 1, MiB, MiB + 1]
    offs = [(0, 0), (1, 1), (3, 7), (16, 5)]
    cases = [(n, so, do) for n in sizes for so, do in offs[: 1 if n > MiB else 4]]
    cases += [(777, 0, 0)] * 20                     # a window beyond the 8 slots
    cases += [(2 * MiB + 4096, 0, 0), (100, 2, 2), (MiB, 0, 0), (5, 0, 0)]   # interleaved protocols
    if rank == 0:
        for i, (n, so, _) in enumerate(cases):
            host = synth.payload(n, 500 + i)
            with torch.cuda.stream(stream):
                src_buf[so:so + n].copy_(torch.from_numpy(host))
            c.send(src_buf[so:so + n], n, 1, tag=1000 + i, stream=stream)
        stream.synchronize()
    elif rank == 1:
        bufs = []
        for i, (n, _, do) in enumerate(cases):
            p = c.alloc(n + 64)
            c.recv(p + do, n, 0, tag=1000 + i, stream=stream)
            bufs.append(p)
        stream.synchronize()
        c.sync()
        for i, ((n, _, do), p) in enumerate(zip(cases, bufs)):
            got = mp_tensor(p + do, n).cpu().numpy()
            exp = synth.payload(n, 500 + i)
            bad = np.nonzero(got != exp)[0]
            assert bad.size == 0, f"eager case {i} (n={n}, dst+{do}): {bad.size} bytes differ, first {bad[:4]}"
            c.free(p)
    dist.barrier()
    c.sync()
    c.close()


def mp_tensor(ptr, n):
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    return mp.as_tensor(ptr, n)


def scenario_coll(rank, world):
    """NEXT f3: mp_alltoall (Bruck, pairwise) and mp_allreduce (K-nomial when
    W is a power of two, ring) through the multi-rank engine against the oracle's MPI
    definitions: Alltoall and the int32 Allreduce exact; fp32 / bf16 sums within the
    rounding bound of W − 1 reassociated additions; in place and out of place."""
    import numpy as np

    from oracle import collectives as OCL
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    BMAX = 300 * 1024 + 5
    send = torch.zeros(world * BMAX + 64, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0)
    rbuf = c.alloc(world * BMAX + 64)
    rview = mp.as_tensor(rbuf, world * BMAX + 64)

    def put(t, arr):
        with torch.cuda.stream(stream):
            t[:arr.nbytes].copy_(torch.from_numpy(arr.view(np.uint8)))
        stream.synchronize()

    def get(t, nbytes):
        stream.synchronize()
        return t[:nbytes].cpu().numpy()

    for algo in (mp.MP_ALGO_BRUCK, mp.MP_ALGO_PAIRWISE):
        for B in (1000, BMAX):
            sends = [np.random.default_rng(97 * s + B + algo).integers(0, 256, world * B, dtype=np.uint8)
                     for s in range(world)]
            put(send, sends[rank])
            c.alltoall(send, rview, B, algo, stream)
            got = get(rview, world * B)
            exp = OCL.alltoall(sends, B)[rank]
            bad = np.nonzero(got != exp)[0]
            assert bad.size == 0, f"alltoall algo {algo} B {B}: {bad.size} bytes differ, first {bad[:4]}"
            dist.barrier()
    algos = [mp.MP_ALGO_RING] + ([mp.MP_ALGO_KNOMIAL] if world & (world - 1) == 0 else [])
    count = 100003
    for algo in algos:
        # int32, out of place (send buffer: any device memory; receive buffer: the heap)
        sends = [np.random.default_rng(31 * s + algo).integers(-2 ** 31, 2 ** 31, count, dtype=np.int64)
                 .astype(np.int32) for s in range(world)]
        put(send, sends[rank])
        c.allreduce(send, rview, count, mp.MP_DT_I32, algo, stream)
        got = get(rview, 4 * count).view(np.int32)
        assert np.array_equal(got, OCL.allreduce_sum(sends).astype(np.int32)), f"allreduce i32 algo {algo}"
        dist.barrier()
        # fp32 and bf16, in place in the heap buffer
        for dt, npdt, eps in ((mp.MP_DT_F32, np.float32, 2.0 ** -24), (mp.MP_DT_BF16, None, 2.0 ** -8)):
            rng = np.random.default_rng(53 * rank + algo + dt)
            x = rng.standard_normal(count).astype(np.float32)
            if npdt is None:   # bf16: the upper 16 bits of the fp32 pattern (round to nearest even)
                u = x.view(np.uint32)
                u = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16).astype(np.uint16)
                arr, vals = u, (u.astype(np.uint32) << 16).view(np.float32)
            else:
                arr, vals = x, x
            allv = [None] * world
            dist.all_gather_object(allv, vals)
            put(rview, arr)
            c.allreduce(rview, rview, count, dt, algo, stream)
            raw = get(rview, arr.nbytes)
            got = raw.view(np.float32) if npdt is not None else (raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32)
            exact = OCL.allreduce_sum(allv)
            bound = (world - 1) * eps * np.sum([np.abs(v.astype(np.float64)) for v in allv], axis=0) * 1.01 + 1e-30
            err = np.abs(got.astype(np.float64) - exact)
            assert (err <= bound).all(), f"allreduce dtype {dt} algo {algo}: max err / bound {np.max(err / bound)}"
            dist.barrier()
    c.sync()
    c.free(rbuf)
    c.close()


def scenario_devsync(rank, world):
    """The relay needs no idle device: relay kernels are launched
    per relayed message by the relay rank's doorbell thread and end with it, so every
    rank may device-synchronise (torch.cuda.synchronize), allocate and load new CUDA
    kernels at any time after mp_init — here between messages and, on the relay rank,
    while a relayed message is in flight.  Payloads bit-exact against the oracle."""
    import numpy as np

    import synth
    from oracle import transfer as X
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0, calibrate=False)
    # CUDA work created only now, after mp_init: a fresh allocation, a generator kernel
    src_buf = torch.empty(8 * MiB, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    ps = c.paths(0, 1)
    np_ = len(ps)
    n = 6 * MiB + 4099
    for i in range(4):
        nb = [0] * np_
        ks = [1] + [0] * (np_ - 1)
        if i % 2 == 0:       # every relay alone, k = 7
            for j in range(1, np_ - 1):
                nb[j] = (n // (np_ - 2)) // 256 * 256
                ks[j] = 7
            nb[-2] += n - sum(nb)
        else:                # direct + relays + host
            for j in range(1, np_):
                nb[j] = 1 * MiB
                ks[j] = 3
            nb[0] = n - sum(nb)
        host = synth.payload(n, 300 + i)
        if rank == 0:
            src = src_buf[:n]
            src.copy_(torch.from_numpy(host))
            torch.cuda.synchronize()
            c.send(src, n, 1, tag=7, cfg=c.make_config(nb, ks, 0, 1), stream=stream)
        elif rank == 1:
            p = c.alloc(n)
            c.recv(p, n, 0, tag=7, stream=stream)
        else:
            # the relay rank device-synchronises while the message may be in flight
            # and launches a kernel it never ran before
            torch.cuda.synchronize()
            x = torch.randint(0, 256, (1 << 20,), dtype=torch.uint8, device="cuda",
                              generator=torch.Generator(device="cuda").manual_seed(i))
            assert int(x.sum().item()) > 0
        torch.cuda.synchronize()   # every rank, device-wide, between messages
        if rank == 1:
            exp = np.zeros(n, dtype=np.uint8)
            X.replay(host, nb, ks, [k for k, _ in ps], 256, exp)
            assert np.array_equal(mp.as_tensor(p, n).cpu().numpy(), exp), f"message {i} mismatch"
            c.free(p)
        c.sync()
        dist.barrier()
    if rank >= 2:
        assert c.launches() >= 1, c.launches()   # relay kernels ran (one serves a burst of messages)
    c.close()


def scenario_bench_plan(rank, world):
    """bench.py --gpus N (config 3) on CPU: rank roles (0 sends, 1 receives, 2.. relay),
    every rank derives the same model config for GPU0 -> GPU1 over direct + relays
    GPU2..GPU{N-1} + host, and the workload label names the executed split."""
    import argparse

    import bench
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    roles = bench.p2p_roles(world)
    assert roles[0] == "sender" and roles[1] == "receiver" and roles[2:] == ["relay"] * (world - 2)
    c = mdist.context_from_dist(model_only=True)
    n = 1 << 30
    r2, cfg = bench.p2p_plan(c, world, n, "b200")
    d = cfg.as_dict()
    assert r2 == roles
    assert d["paths"] == [(0, -1)] + [(1, r) for r in range(2, world)] + [(2, -1)], d["paths"]
    assert sum(d["bytes"]) == n
    out = [None] * world
    dist.all_gather_object(out, (d["bytes"], d["chunks"]))
    assert all(o == out[0] for o in out)
    args = argparse.Namespace(size=n, mode="b200", workload="config3")
    w = bench.workload_config(args, world, d)
    assert w["paths"] == f"direct+{world - 2}relay+host" and w["selected"] == bench.split_label(d)
    assert w["parallelism"] == f"p2p-1pair+{world - 2}relays"
    c.close()
    # one GPU per rank, checked across the ranks by GPU UUID: with fewer GPUs than ranks
    # (none on the CPU box) every rank refuses, none proceeds alone
    n_gpu = torch.cuda.device_count() if torch.cuda.is_available() else 0
    if n_gpu >= world:
        assert bench.rank_device(rank, world) == rank
    else:
        try:
            bench.rank_device(rank, world)
            raise AssertionError("rank_device accepted fewer GPUs than ranks")
        except SystemExit as e:
            assert "one GPU per rank" in str(e)


def scenario_relay_burst(rank, world):
    """Doorbell and lingering-relay bookkeeping under load: 160 relayed messages rank 0
    → rank 1 through relay rank 2 (2.5 doorbell rings of 64), windows of 8 in flight,
    alternating co-aligned and misaligned sources (a lingering relay kernel switches
    between its streamed and per-chunk paths message by message), with pauses longer
    than the linger between some windows (the host thread relaunches).  Every message
    bit-exact against the oracle replay."""
    import time

    import numpy as np

    import synth
    from oracle import transfer as X
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4,
                                timeout_s=60.0, calibrate=False)
    ps = c.paths(0, 1)
    n = 1 * MiB + 4099
    W = 8
    src_buf = torch.empty(W * (n + 64), dtype=torch.uint8, device="cuda")
    bufs = [c.alloc(n) for _ in range(W)] if rank == 1 else []
    nb = [0] * len(ps)
    nb[1] = n
    ks = [1] + [0] * (len(ps) - 1)
    ks[1] = 3
    cfg = c.make_config(nb, ks, 0, 1)
    for win in range(20):
        payloads = [synth.payload(n, 1000 + win * W + i) for i in range(W)]
        if rank == 0:
            views = []
            for i in range(W):
                off = i * (n + 64) + (0 if (win + i) % 2 == 0 else 7)  # co-aligned, then misaligned
                v = src_buf[off:off + n]
                v.copy_(torch.from_numpy(payloads[i]))
                views.append(v)
            torch.cuda.synchronize()
            for i in range(W):
                c.send(views[i], n, 1, tag=win * W + i, cfg=cfg, stream=stream)
            stream.synchronize()
        elif rank == 1:
            for i in range(W):
                c.recv(bufs[i], n, 0, tag=win * W + i, stream=stream)
            stream.synchronize()
            for i in range(W):
                exp = np.zeros(n, dtype=np.uint8)
                X.replay(payloads[i], nb, ks, [k for k, _ in ps], 256, exp)
                assert np.array_equal(mp.as_tensor(bufs[i], n).cpu().numpy(), exp), f"window {win} message {i}"
        if win % 5 == 4:
            time.sleep(0.002)  # > the 200 µs linger: the relay kernel ends, the host thread relaunches
        dist.barrier()
    c.sync()
    for b in bufs:
        c.free(b)
    c.close()


def scenario_full_size(rank, world):
    """BASELINE.json config 3 at full size through the multi-rank engine, in bench.py's
    launch configuration (default slots / lanes / heap, deep staged pipelines): one
    1 GiB + 4099-byte message rank 0 → rank 1 with the B200-mode pick, then with the
    paper-mode pick (every path: direct, relays 2.., host) and every path forced at
    once; payloads compared whole on the device against the source (O1: dst == src)."""
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    n = (1 << 30) + 4099
    stream = torch.cuda.Stream()
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                        generator=torch.Generator(device="cuda").manual_seed(20251116)) if rank in (0, 1) else None
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=n + 64 * MiB, timeout_s=120.0, calibrate=False)
    rbuf = c.alloc(n) if rank == 1 else None
    ps = c.paths(0, 1)
    cfgs = []
    for mode in (mp.MP_MODEL_B200, mp.MP_MODEL_PAPER):
        c.set_options(mode=mode)
        cfgs.append(c.select(0, 1, n).as_dict())
    nb = [0] * len(ps)
    for j in range(1, len(ps)):
        nb[j] = (64 if ps[j][0] == 1 else 16) * MiB + 256 * j
    nb[0] = n - sum(nb)
    cfgs.append({"bytes": nb, "chunks": [1] + [8] * (len(ps) - 1)})
    for i, d in enumerate(cfgs):
        if rank == 0:
            c.send(src, n, 1, tag=i, cfg=c.make_config(d["bytes"], d["chunks"], 0, 1), stream=stream)
            stream.synchronize()
        elif rank == 1:
            view = mp.as_tensor(rbuf, n)
            view.zero_()
            torch.cuda.synchronize()
            c.recv(rbuf, n, 0, tag=i, stream=stream)
            stream.synchronize()
            assert torch.equal(view, src), f"config {i}: {d['bytes']}"
        dist.barrier()
    c.sync()
    if rbuf:
        c.free(rbuf)
    c.close()


def scenario_wake(rank, world):
    """Reading C28: mp_calibrate_wake measures each relay rank's start time and every
    GPU-staged path via that relay carries it in every pair model (all ranks agree);
    the MPX_RELAY_WAKE_US override installs its value exactly; relayed messages stay
    bit-exact and the B200 pick's prediction includes the wake."""
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    stream = torch.cuda.Stream()
    n = 8 * MiB + 4099
    src = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                        generator=torch.Generator(device="cuda").manual_seed(7)) if rank == 0 else None
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=64 * MiB, timeout_s=60.0, calibrate=False)
    c.calibrate(sizes=[4 * MiB, 8 * MiB, 16 * MiB], reps=2)   # Step 1, then the wake probe
    wakes = {}
    for s_ in range(world):
        for d_ in range(world):
            if s_ == d_:
                continue
            paths, prm, _ = c.get_model(s_, d_)
            for (kind, via), p in zip(paths, prm):
                if kind == mp.MP_PATH_GPU:
                    # every rank on one GPU: µs under MPS, a scheduling time slice (ms) without
                    assert 0.0 <= p["wake"] < 0.1, (s_, d_, via, p["wake"])
                    assert wakes.setdefault(via, p["wake"]) == p["wake"]   # one value per relay
                else:
                    assert p["wake"] == 0.0
    allw = [None] * world
    dist.all_gather_object(allw, wakes)
    assert all(w == allw[0] for w in allw), allw
    print(f"rank {rank}: measured relay wakes [us] " + str({k: round(v * 1e6, 2) for k, v in wakes.items()}),
          flush=True)
    os.environ["MPX_RELAY_WAKE_US"] = "50"
    c.calibrate_wake()
    del os.environ["MPX_RELAY_WAKE_US"]
    paths, prm, _ = c.get_model(0, 1)
    for (kind, _), p in zip(paths, prm):
        assert p["wake"] == (50e-6 if kind == mp.MP_PATH_GPU else 0.0)
    c.set_options(mode=mp.MP_MODEL_B200)
    nb = [0] * len(paths)
    nb[1] = n
    ks = [1] + [0] * (len(paths) - 1)
    ks[1] = 4
    cfg = c.make_config(nb, ks, 0, 1)
    p1 = prm[1]
    s2 = p1["eps"] + p1["alpha2"] + n / 4 / p1["beta2"]
    assert c.predict(0, 1, n, cfg) >= 50e-6 + 4 * s2 - 1e-12
    rbuf = c.alloc(n) if rank == 1 else None
    if rank == 0:
        c.send(src, n, 1, tag=5, cfg=cfg, stream=stream)
        c.send(src, n, 1, tag=6, cfg=None, stream=stream)
        stream.synchronize()
        dist.send(torch.tensor([1]), 1)
    elif rank == 1:
        view = mp.as_tensor(rbuf, n)
        ref = torch.empty(n, dtype=torch.uint8, device="cuda")
        for t in (5, 6):
            view.zero_()
            torch.cuda.synchronize()
            c.recv(rbuf, n, 0, tag=t, stream=stream)
            stream.synchronize()
            if t == 5:
                ref.copy_(view)
        dist.recv(torch.tensor([0]), 0)
        exp = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda",
                            generator=torch.Generator(device="cuda").manual_seed(7))
        assert torch.equal(ref, exp) and torch.equal(view, exp)
    dist.barrier()
    c.sync()
    if rbuf:
        c.free(rbuf)
    c.close()


def scenario_bell_flow(rank, world):
    """Many relayed messages in flight: rank 0 sends 56 relayed messages to rank 1 and 56
    to rank 3, every one through relay rank 2 on its own stream (112 streams), receivers
    posting on 56 streams each, the later messages' streams delayed least.  More doorbells than the relay's
    ring holds (64: the gates' acknowledgement wait), and send kernels that become
    resident out of ring order (the cross-stream ring order).  Every message bit-exact."""
    from paper_conf_sc_sojoodiasfga25_b200 import dist as mdist
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    torch.cuda.set_device(DEV)
    n, M = 1 * MiB + 4099, 56
    gen = torch.Generator(device="cuda").manual_seed(11)
    src = torch.randint(0, 256, (2 * M, n), dtype=torch.uint8, device="cuda", generator=gen)
    torch.cuda.synchronize()
    c = mdist.context_from_dist(device=DEV, heap_bytes=M * (n + 4096) + 8 * MiB, timeout_s=60.0, calibrate=False)
    streams = [torch.cuda.Stream() for _ in range(2 * M)]
    peers = (1, 3)
    if rank == 0:
        for i in range(2 * M):
            d = peers[i % 2]
            ps = c.paths(0, d)
            idx = next(j for j, (k, via) in enumerate(ps) if k == mp.MP_PATH_GPU and via == 2)
            nb = [0] * len(ps)
            nb[idx] = n
            ks = [1] + [0] * (len(ps) - 1)
            ks[idx] = 1
            c.send(src[i], n, d, tag=i, cfg=c.make_config(nb, ks, 0, d), stream=streams[i])
        torch.cuda.synchronize()
    elif rank in peers:
        bufs = [c.alloc(n) for _ in range(M)]
        mine = [i for i in range(2 * M) if peers[i % 2] == rank]
        # posted in order (matching is FIFO per pair), but each stream first sleeps the
        # longer the earlier its message: the later messages' clear-to-sends arrive first,
        # so their gates fire (and their send kernels become resident) before the earlier ones'
        for j in range(M):
            with torch.cuda.stream(streams[j]):
                torch.cuda._sleep(40000 * (M - j))
            c.recv(bufs[j], n, 0, tag=mine[j], stream=streams[j])
        torch.cuda.synchronize()
        c.sync()  # sticky device errors (timeout, mismatch) first
        for j, i in enumerate(mine):
            assert torch.equal(mp.as_tensor(bufs[j], n), src[i]), f"message {i}"
        for b in bufs:
            c.free(b)
    dist.barrier()
    c.sync()
    c.close()


def main():
    rank, world, port, scen = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
    import faulthandler
    faulthandler.enable()
    faulthandler.dump_traceback_later(int(os.environ.get("MPX_TEST_STACKS_S", "280")), exit=False)
    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        {"gloo_model": scenario_gloo_model, "engine": scenario_engine,
         "faults": scenario_faults, "register": scenario_register, "coll": scenario_coll,
         "eager": scenario_eager, "devsync": scenario_devsync,
         "bench_plan": scenario_bench_plan, "relay_burst": scenario_relay_burst,
         "full_size": scenario_full_size, "wake": scenario_wake,
         "bell_flow": scenario_bell_flow}[scen](rank, world)
        dist.barrier()
        dist.destroy_process_group()
    except BaseException:
        import traceback
        traceback.print_exc()
        sys.stdout.flush()
        sys.stderr.flush()
        os._exit(1)  # skip interpreter teardown (no collective finalisers at exit)
    print(f"rank {rank} ok", flush=True)


if __name__ == "__main__":
    main()
