"""The multi-rank engine on ONE GPU as an emulated world (include/mp.h: mp_init_emulated,
mp_emu_run): every rank is a context of this process, and every rank's kernels — the
send gate and send CTAs, the receive CTAs, the relay kernels a relay rank's service
thread would launch, the eager kernels — run as CTA ranges of ONE cooperative launch.
Ranks whose kernels wait on one another are then co-resident by construction, never
separate launches sharing the GPU (the B200 profiling guide's rule when there are fewer
GPUs than ranks).  Payloads are checked byte for byte against the oracle's reference
transfer (oracle/transfer.py: replay of the split)."""
import numpy as np
import pytest

import synth
from oracle import transfer as X

pytestmark = pytest.mark.gpu

MiB = 1 << 20


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    torch.cuda.set_device(0)
    return torch


def world(w, **kw):
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    args = dict(device=0, heap_bytes=96 * MiB, slot_bytes=1 * MiB, slots=2, relay_ctas=4, timeout_s=20.0)
    args.update(kw)
    return mp.EmulatedWorld(w, **args)


def expected(host, nb, ks, ps):
    exp = np.zeros(len(host), dtype=np.uint8)
    if nb is None:
        exp[:] = host
    else:
        X.replay(host, nb, ks, [k for k, _ in ps], 256, exp)
    return exp


def fill(torch, n, seed):
    host = synth.payload(n, seed)
    return host, torch.from_numpy(host).cuda()


def cases_for(ps, n):
    """Direct only, one relay alone (k = 5), host alone (k = 4), every path at once."""
    np_ = len(ps)
    out = [([n] + [0] * (np_ - 1), [1] + [0] * (np_ - 1))]
    if np_ > 2:
        nb, ks = [0] * np_, [1] + [0] * (np_ - 1)
        nb[1], ks[1] = n, 5
        out.append((nb, ks))
    nb, ks = [0] * np_, [1] + [0] * (np_ - 1)
    nb[-1], ks[-1] = n, 4
    out.append((nb, ks))
    nb = [0] + [256 * 1024] * (np_ - 1)
    nb[0] = n - sum(nb)
    out.append((nb, [1] + [2] * (np_ - 1)))
    return out


@pytest.mark.parametrize("w", [2, 3, 4])
def test_emulated_pair_every_path_kind_bit_exact(torch_cuda, w):
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(w) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        assert len(ps) == w  # direct + (w - 2) relays + host
        n = 3 * MiB + 4099
        for i, (nb, ks) in enumerate(cases_for(ps, n) + [(None, None)]):
            host, src = fill(torch, n, i)
            dst = c1.alloc(n)
            mp.as_tensor(dst, n).zero_()
            torch.cuda.synchronize()
            c0.send(src, n, 1, tag=100 + i, cfg=c0.make_config(nb, ks, 0, 1) if nb else None)
            c1.recv(dst, n, 0, tag=100 + i)
            W.run()
            got = mp.as_tensor(dst, n).cpu().numpy()
            assert np.array_equal(got, expected(host, nb, ks, ps)), f"world {w} case {i} {nb} {ks}"
            c1.free(dst)
        assert c0.launches() > 0


def test_emulated_windows_ring_wrap_bidirectional_eager_zero(torch_cuda):
    """One run holding a window of 4 messages each way between ranks 0 and 1 (every path,
    k = 2 on 2-slot rings: the relay and host rings wrap twice; the relay role serves
    four doorbells through the lingering relay's next-message decisions), plus an eager
    message, a zero-byte message and a message relayed 2 -> 3 through ranks 0 and 1."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(4) as W:
        c = W.ctx
        ps = c[0].paths(0, 1)
        n = 2 * MiB + 77
        nb = [0] + [256 * 1024] * (len(ps) - 1)
        nb[0] = n - sum(nb)
        ks = [1] + [2] * (len(ps) - 1)
        checks = []
        for s, d in ((0, 1), (1, 0)):
            for m in range(4):
                host, src = fill(torch, n, 10 * s + m)
                dst = c[d].alloc(n)
                checks.append((d, dst, n, expected(host, nb, ks, c[s].paths(s, d)), src))
                c[s].send(src, n, d, tag=m, cfg=c[s].make_config(nb, ks, s, d))
                c[d].recv(dst, n, s, tag=m)
        # eager (<= 1 MiB: no rendezvous) and zero-byte messages 2 -> 3
        host_e, src_e = fill(torch, 300 * 1000 + 5, 99)
        dst_e = c[3].alloc(len(host_e))
        c[2].send(src_e, len(host_e), 3, tag=7)
        c[3].recv(dst_e, len(host_e), 2, tag=7)
        c[2].send(src_e, 0, 3, tag=8)
        c[3].recv(dst_e, 0, 2, tag=8)
        checks.append((3, dst_e, len(host_e), host_e, src_e))
        # 2 -> 3 through both other ranks as relays, concurrently with the 0 <-> 1 windows
        ps23 = c[2].paths(2, 3)
        nb23 = [0] * len(ps23)
        ks23 = [1] + [0] * (len(ps23) - 1)
        for i, (k, v) in enumerate(ps23):
            if k == 1:
                nb23[i], ks23[i] = MiB, 3
        n23 = sum(nb23) + 12345
        nb23[0] = 12345
        host23, src23 = fill(torch, n23, 123)
        dst23 = c[3].alloc(n23)
        c[2].send(src23, n23, 3, tag=9, cfg=c[2].make_config(nb23, ks23, 2, 3))
        c[3].recv(dst23, n23, 2, tag=9)
        checks.append((3, dst23, n23, expected(host23, nb23, ks23, ps23), src23))
        torch.cuda.synchronize()
        W.run()
        for j, (d, p, nn, exp, _) in enumerate(checks):
            assert np.array_equal(mp.as_tensor(p, nn).cpu().numpy(), exp), f"message {j}"
        # the pairs' sequence state carries over: a second run on the same world
        host, src = fill(torch, n, 55)
        dst = c[1].alloc(n)
        c[0].send(src, n, 1, tag=1, cfg=c[0].make_config(nb, ks, 0, 1))
        c[1].recv(dst, n, 0, tag=1)
        W.run()
        assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), expected(host, nb, ks, ps))


def test_emulated_config3_shape_full_relay_fan(torch_cuda):
    """BASELINE config 3's shape on one GPU: rank 0 -> rank 1 over direct + 6 relay
    ranks + the pinned host path (world 8), every path carrying bytes, 64 MiB + 4099 B."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(8, heap_bytes=80 * MiB, slot_bytes=4 * MiB, slots=2) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        assert [k for k, _ in ps] == [0] + [1] * 6 + [2]
        n = 64 * MiB + 4099
        nb = [0] + [6 * MiB] * 6 + [2 * MiB]
        nb[0] = n - sum(nb)
        ks = [1] + [4] * 6 + [3]
        host, src = fill(torch, n, 3)
        dst = c1.alloc(n)
        c0.send(src, n, 1, tag=3, cfg=c0.make_config(nb, ks, 0, 1))
        c1.recv(dst, n, 0, tag=3)
        torch.cuda.synchronize()
        W.run()
        assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), expected(host, nb, ks, ps))


def test_emulated_all_pairs_concurrent(torch_cuda):
    """BASELINE config 5's shape (world 4): every ordered pair sends at once, each over
    direct + both other ranks as relays + host, in one grid."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(4) as W:
        c = W.ctx
        n = 1 * MiB + 2 * 256 * 1024 + 513
        checks = []
        for s in range(4):
            for d in range(4):
                if s == d:
                    continue
                ps = c[s].paths(s, d)
                nb = [0] + [256 * 1024] * (len(ps) - 1)
                nb[0] = n - sum(nb)
                ks = [1] + [2] * (len(ps) - 1)
                host, src = fill(torch, n, 16 * s + d)
                dst = c[d].alloc(n)
                c[s].send(src, n, d, tag=s, cfg=c[s].make_config(nb, ks, s, d))
                c[d].recv(dst, n, s, tag=s)
                checks.append((d, dst, expected(host, nb, ks, ps), src))
        torch.cuda.synchronize()
        W.run()
        for j, (d, p, exp, _) in enumerate(checks):
            assert np.array_equal(mp.as_tensor(p, n).cpu().numpy(), exp), f"pair message {j}"


def test_emulated_faults_reported(torch_cuda):
    """A tag mismatch is MP_ERR_MISMATCH; a send nobody receives is MP_ERR_TIMEOUT —
    both from the device, neither hangs; the unsupported calls say so."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(3, timeout_s=2.0) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        n = 2 * MiB
        _, src = fill(torch, n, 1)
        dst = c1.alloc(n)
        c0.send(src, n, 1, tag=1)
        c1.recv(dst, n, 0, tag=2)
        with pytest.raises(mp.MPError) as e:
            W.run()
        assert e.value.status == mp.MP_ERR_MISMATCH
        with pytest.raises(mp.MPError) as e:
            c0.calibrate()
        assert e.value.status == mp.MP_ERR_UNSUPPORTED
    with world(2, timeout_s=1.0) as W:
        _, src = fill(torch, 2 * MiB, 1)
        W.ctx[0].send(src, 2 * MiB, 1, tag=1)
        with pytest.raises(mp.MPError) as e:
            W.run()
        assert e.value.status == mp.MP_ERR_TIMEOUT


def test_emulated_relay_burst_doorbell_wrap_and_eager_wrap(torch_cuda):
    """160 relayed messages rank 0 -> rank 1 through relay rank 2 in 20 runs of 8 (the
    doorbell ring of 64 and the relay's decision ring wrap 2.5 times; each run's relay
    role serves 8 doorbells), sources alternately co-aligned and misaligned (streamed
    and per-chunk relay lanes, message by message), plus one eager message per run
    (the 8 eager slots wrap)."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    with world(3) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        n, M = 1 * MiB + 4099, 8
        nb = [0] * len(ps)
        nb[1] = n
        ks = [1] + [0] * (len(ps) - 1)
        ks[1] = 3
        cfg = c0.make_config(nb, ks, 0, 1)
        src_buf = torch.empty(M * (n + 64), dtype=torch.uint8, device="cuda")
        bufs = [c1.alloc(n) for _ in range(M)]
        ne = 40000 + 3
        ebuf = c1.alloc(ne)
        for run in range(20):
            payloads = [synth.payload(n, 1000 + run * M + i) for i in range(M)]
            for i in range(M):
                off = i * (n + 64) + (0 if (run + i) % 2 == 0 else 7)
                v = src_buf[off:off + n]
                v.copy_(torch.from_numpy(payloads[i]))
                c0.send(v, n, 1, tag=run * M + i, cfg=cfg)
                c1.recv(bufs[i], n, 0, tag=run * M + i)
            he, se = fill(torch, ne, 5000 + run)
            c0.send(se, ne, 1, tag=-1 - run)
            c1.recv(ebuf, ne, 0, tag=-1 - run)
            torch.cuda.synchronize()
            W.run()
            for i in range(M):
                assert np.array_equal(mp.as_tensor(bufs[i], n).cpu().numpy(), expected(payloads[i], nb, ks, ps)), \
                    f"run {run} message {i}"
            assert np.array_equal(mp.as_tensor(ebuf, ne).cpu().numpy(), he), f"run {run} eager"


def test_emulated_config3_full_size_default_launch_config(torch_cuda):
    """BASELINE config 3's message size (1 GiB + 4099 B) in the engine's default launch
    configuration (4 slots of 32 MiB, 16 lanes per stage group, deep staged pipelines):
    every path at once and direct-only, world 3, compared on the device against the
    oracle's replay."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    n = (1 << 30) + 4099
    with mp.EmulatedWorld(3, device=0, heap_bytes=n + 64 * MiB, timeout_s=60.0) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        host = synth.payload(n, 33)
        src = torch.from_numpy(host).cuda()
        dst = c1.alloc(n)
        for nb, ks in (([n - 448 * MiB, 320 * MiB, 128 * MiB], [1, 12, 5]), ([n, 0, 0], [1, 0, 0])):
            mp.as_tensor(dst, n).zero_()
            torch.cuda.synchronize()
            c0.send(src, n, 1, tag=0, cfg=c0.make_config(nb, ks, 0, 1))
            c1.recv(dst, n, 0, tag=0)
            W.run()
            exp = torch.from_numpy(expected(host, nb, ks, ps)).cuda()
            assert torch.equal(mp.as_tensor(dst, n), exp), (nb, ks)
            del exp


def _install(ctx, src, dst, tbl, port):
    ctx.set_model(src, dst, [(t["kind"], t["via"]) for t in tbl],
                  [{k: (0.0 if k == "beta2" and t["kind"] == 0 else t[k])
                    for k in ("alpha", "beta", "alpha2", "beta2", "eps", "c", "sigma", "w")} for t in tbl], port)


@pytest.mark.parametrize("mode", ["paper", "b200"])
def test_emulated_config2_model_selected_multipath_split(torch_cuda, mode):
    """BASELINE config 2 (64 MiB, GPU0 -> GPU1, direct + 2 GPU relays): an NVLink-like
    parameter table (synth.topology) installed on the sender; the library's pick over
    direct + both relays (host path masked out) equals the oracle's (bytes, chunks,
    t_pred within 1e-9), and that multi-path split moves bit-exact through the emulated
    world's kernels."""
    torch = torch_cuda
    from oracle import model as OM
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    n = 64 * MiB
    port = dict(alpha=1.5e-6, beta=850e9)
    with world(4, heap_bytes=n + 8 * MiB, slot_bytes=8 * MiB, slots=4) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        o = c0.get_options()
        o["mode"] = mp.MP_MODEL_PAPER if mode == "paper" else mp.MP_MODEL_B200
        c0.set_options(**o)
        ps = c0.paths(0, 1)
        for seed in (3, 8):
            tbl = synth.topology(seed, 2, host=True)
            assert [(t["kind"], t["via"]) for t in tbl] == ps
            _install(c0, 0, 1, tbl, port)
            d = c0.select(0, 1, n, 0b0111).as_dict()
            ref = OM.select(n, [OM.Path(**t) for t in tbl],
                            OM.Options(mode=o["mode"], stagger=bool(o["stagger"]), align=o["align"],
                                       c_min=o["c_min"], k_max=o["k_max"], slot_bytes=o["slot_bytes"]),
                            OM.Port(**port), path_mask=[True, True, True, False])
            assert d["bytes"] == list(ref.bytes) and d["chunks"] == list(ref.chunks), (d, ref)
            assert abs(d["t_pred"] - ref.t_pred) <= 1e-9 * ref.t_pred
            assert sum(d["bytes"][1:3]) > 0, "an NVLink-like table puts bytes on the relays"
            host, src = fill(torch, n, seed)
            dst = c1.alloc(n)
            c0.send(src, n, 1, tag=seed, cfg=c0.make_config(d["bytes"], d["chunks"], 0, 1))
            c1.recv(dst, n, 0, tag=seed)
            torch.cuda.synchronize()
            W.run()
            assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), expected(host, d["bytes"], d["chunks"], ps))
            c1.free(dst)


def test_emulated_config1_forced_split(torch_cuda):
    """BASELINE config 1: 1 MiB GPU0 -> GPU1, direct + 1 relay, 4 chunks, θ = (3/4, 1/4)
    (SURVEY §8(d)), world 3 (relay rank 2, no host path)."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    n = 1 << 20
    with world(3, host_path=0) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        assert [k for k, _ in ps] == [0, 1]
        nb, ks = [3 * n // 4, n // 4], [1, 4]
        host, src = fill(torch, n, 11)
        dst = c1.alloc(n)
        c0.send(src, n, 1, tag=1, cfg=c0.make_config(nb, ks, 0, 1))
        c1.recv(dst, n, 0, tag=1)
        W.run()
        assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), expected(host, nb, ks, ps))


@pytest.mark.parametrize("stages", ["4", "6"])
def test_emulated_both_staged_pipeline_depths(torch_cuda, monkeypatch, stages):
    """The send / receive / relay bodies at each staged-pipeline depth (MPX_STAGES: the
    real launches pick one per launch; the emulated grid runs every role at one):
    every path kind at world 3, co-aligned and misaligned sources."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    monkeypatch.setenv("MPX_STAGES", stages)
    with world(3, relay_ctas=8, slot_bytes=2 * MiB) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        n = 5 * MiB + 333
        buf = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
        for i, (nb, ks) in enumerate(cases_for(ps, n)):
            for shift in (0, 5):
                host = synth.payload(n, 40 + i)
                src = buf[shift:shift + n]
                src.copy_(torch.from_numpy(host))
                dst = c1.alloc(n)
                c0.send(src, n, 1, tag=i, cfg=c0.make_config(nb, ks, 0, 1))
                c1.recv(dst, n, 0, tag=i)
                torch.cuda.synchronize()
                W.run()
                assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), expected(host, nb, ks, ps)), (stages, i, shift)
                c1.free(dst)


@pytest.mark.parametrize("w", [2, 3, 4])
def test_emulated_collectives_against_mpi_definitions(torch_cuda, w):
    """NEXT f3 in the emulated world: mp_emu_alltoall (Bruck, pairwise) and
    mp_emu_allreduce (ring; K-nomial when W is a power of two) — the same plans and
    per-step multi-path configs as mp_alltoall / mp_allreduce, each step one
    cooperative grid — against the oracle's MPI definitions: Alltoall and the int32
    Allreduce exact; fp32 / bf16 sums within the rounding bound of W - 1 reassociated
    additions; out of place and in place."""
    torch = torch_cuda
    from oracle import collectives as OCL
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    BMAX = 300 * 1024 + 5
    with world(w) as W:
        sends = [torch.zeros(w * BMAX + 64, dtype=torch.uint8, device="cuda") for _ in range(w)]
        rbufs = [W.ctx[r].alloc(w * BMAX + 64) for r in range(w)]
        rviews = [mp.as_tensor(rbufs[r], w * BMAX + 64) for r in range(w)]

        def put(t, arr):
            t[:arr.nbytes].copy_(torch.from_numpy(arr.view(np.uint8)))
            torch.cuda.synchronize()

        for algo in (mp.MP_ALGO_BRUCK, mp.MP_ALGO_PAIRWISE):
            for B in (1000, BMAX):
                data = [np.random.default_rng(97 * s + B + algo).integers(0, 256, w * B, dtype=np.uint8)
                        for s in range(w)]
                for r in range(w):
                    put(sends[r], data[r])
                W.alltoall(sends, rviews, B, algo)
                exp = OCL.alltoall(data, B)
                for r in range(w):
                    got = rviews[r][:w * B].cpu().numpy()
                    assert np.array_equal(got, exp[r]), f"alltoall algo {algo} B {B} rank {r}"
        algos = [mp.MP_ALGO_RING] + ([mp.MP_ALGO_KNOMIAL] if w & (w - 1) == 0 else [])
        count = 100003
        for algo in algos:
            data = [np.random.default_rng(31 * s + algo).integers(-2 ** 31, 2 ** 31, count, dtype=np.int64)
                    .astype(np.int32) for s in range(w)]
            for r in range(w):
                put(sends[r], data[r])
            W.allreduce(sends, rviews, count, mp.MP_DT_I32, algo)
            exp = OCL.allreduce_sum(data).astype(np.int32)
            for r in range(w):
                got = rviews[r][:4 * count].cpu().numpy().view(np.int32)
                assert np.array_equal(got, exp), f"allreduce i32 algo {algo} rank {r}"
            for dt, eps in ((mp.MP_DT_F32, 2.0 ** -24), (mp.MP_DT_BF16, 2.0 ** -8)):
                vals, arrs = [], []
                for r in range(w):
                    x = np.random.default_rng(53 * r + algo + dt).standard_normal(count).astype(np.float32)
                    if dt == mp.MP_DT_BF16:  # round to nearest even on the upper 16 bits
                        u = x.view(np.uint32)
                        u = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16).astype(np.uint16)
                        arrs.append(u)
                        vals.append((u.astype(np.uint32) << 16).view(np.float32))
                    else:
                        arrs.append(x)
                        vals.append(x)
                    put(rviews[r], arrs[r])
                W.allreduce(rviews, rviews, count, dt, algo)  # in place
                exact = OCL.allreduce_sum(vals)
                bound = (w - 1) * eps * np.sum([np.abs(v.astype(np.float64)) for v in vals], axis=0) * 1.01 + 1e-30
                for r in range(w):
                    raw = rviews[r][:arrs[r].nbytes].cpu().numpy()
                    got = raw.view(np.float32) if dt == mp.MP_DT_F32 else \
                        (raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32)
                    err = np.abs(got.astype(np.float64) - exact)
                    assert (err <= bound).all(), f"allreduce dtype {dt} algo {algo} rank {r}: {np.max(err / bound)}"


def test_emulated_registered_regions(torch_cuda):
    """mp_register in the emulated world (mp_emu_register): receives into arbitrary torch
    tensors — two views of one allocation on rank 1, then one tensor per rank in a ring,
    all ring messages in one grid — over every path at once, bit-exact against the
    oracle replay, bytes outside the views untouched; a deregistered region is
    refused; region ids are reused."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    w = 3
    with world(w, heap_bytes=16 * MiB) as W:
        c = W.ctx
        big = torch.zeros(16 * MiB, dtype=torch.uint8, device="cuda")
        rings = [torch.zeros(4 * MiB, dtype=torch.uint8, device="cuda") for _ in range(w)]
        va, vb = big[MiB + 256: 9 * MiB], big[10 * MiB: 15 * MiB]
        ida = W.register([None, va, None])
        idb = W.register([None, vb, None])
        idr = W.register(rings)
        assert len({ida[0], idb[0], idr[0]}) == 3 and ida == [ida[0]] * w
        ps = c[0].paths(0, 1)
        na = 3 * MiB + 4099
        nb = [256 * 1024] * len(ps)
        nb[0] = na - 256 * 1024 * (len(ps) - 1)
        ks = [1] + [2] * (len(ps) - 1)
        for case, (view, n, cb, ck) in enumerate([(va, na, nb, ks), (vb, 5 * MiB, None, None)]):
            host, src = fill(torch, n, 60 + case)
            c[0].send(src, n, 1, tag=300 + case, cfg=c[0].make_config(cb, ck, 0, 1) if cb else None)
            c[1].recv(view[:n], n, 0, tag=300 + case)
            W.run()
            assert np.array_equal(view[:n].cpu().numpy(), expected(host, cb, ck, ps)), f"region case {case}"
        outside = torch.cat([big[:MiB + 256], big[9 * MiB:10 * MiB], big[15 * MiB:]])
        assert int(outside.count_nonzero()) == 0, "bytes outside the registered views were written"
        n = 2 * MiB + 333
        srcs = [fill(torch, n, 70 + r) for r in range(w)]
        for r in range(w):
            nxt, prv = (r + 1) % w, (r - 1) % w
            c[r].recv(rings[r][4096 + 17: 4096 + 17 + n], n, prv, tag=400)
            c[r].send(srcs[r][1], n, nxt, tag=400)
        W.run()
        for r in range(w):
            assert np.array_equal(rings[r][4096 + 17: 4096 + 17 + n].cpu().numpy(), srcs[(r - 1) % w][0]), f"ring {r}"
        for ids in (ida, idb, idr):
            W.deregister(ids)
        with pytest.raises(mp.MPError):
            c[1].recv(va[:MiB], MiB, 0, tag=1)
        assert W.register(rings) == ida  # ids are reused
        W.deregister(ida)


def test_emulated_doorbell_flow_control_one_grid(torch_cuda, monkeypatch):
    """72 relayed messages from rank 0 through relay rank 3, all in flight in ONE grid
    (alternately to ranks 1 and 2: 36 per pair, within the 64 outstanding messages a
    pair's clear-to-send ring holds; one lane per stage group, 2-slot rings): more than
    the 64-entry doorbell ring of (sender, relay), so the gates of messages 64.. wait for
    the relay role to acknowledge doorbells 0.. (flow control) while it serves all 72 in
    doorbell order; every message bit-exact."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    M = 72
    monkeypatch.setenv("MPX_EAGER", "0")  # every message takes the rendezvous (and its relay)
    with world(4, relay_ctas=1, host_path=0, slot_bytes=256 * 1024, slots=2, heap_bytes=64 * MiB) as W:
        c = W.ctx
        n = 192 * 1024 + 40
        checks = []
        for m in range(M):
            d = 1 + m % 2
            ps = c[0].paths(0, d)
            nb, ks = [0] * len(ps), [1] + [0] * (len(ps) - 1)
            i = ps.index((1, 3))
            nb[0], nb[i], ks[i] = 40, n - 40, 1
            host, src = fill(torch, n, 500 + m)
            dst = c[d].alloc(n)
            c[0].send(src, n, d, tag=m, cfg=c[0].make_config(nb, ks, 0, d))
            c[d].recv(dst, n, 0, tag=m)
            checks.append((dst, expected(host, nb, ks, ps), src))
        torch.cuda.synchronize()
        W.run()
        for m, (dst, exp, _) in enumerate(checks):
            assert np.array_equal(mp.as_tensor(dst, n).cpu().numpy(), exp), m


def test_emulated_random_splits_misaligned_with_canaries(torch_cuda):
    """Randomised multi-rank parity (seeded): 24 messages rank 0 -> rank 1 at world 4 with
    random sizes (ragged), random shares over direct / relay 2 / relay 3 / host (any of
    them possibly empty, shares not multiples of A), random chunk counts up to the slot
    limit, and source and destination offsets 0-15 B (co-aligned or not: streamed and
    per-chunk lanes); each payload equal to the oracle replay, 4 KiB canaries on both
    sides of the destination untouched."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    rng = np.random.default_rng(20251018)
    CAN = 4096
    with world(4, slot_bytes=2 * MiB, heap_bytes=64 * MiB) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        ps = c0.paths(0, 1)
        kinds = [k for k, _ in ps]
        sbuf = torch.empty(26 * MiB, dtype=torch.uint8, device="cuda")
        base = c1.alloc(26 * MiB + 2 * CAN + 64)
        dview = mp.as_tensor(base, 26 * MiB + 2 * CAN + 64)
        done = 0
        for case in range(24):
            n = int(rng.integers(1 * MiB, 24 * MiB))
            nb = [0] * len(ps)
            ks = [1] + [0] * (len(ps) - 1)
            left = n
            for i in range(1, len(ps)):
                if rng.random() < 0.75 and left > 1024:
                    b = int(rng.integers(300, max(301, min(left, 6 * MiB))))
                    U = b // 256
                    kmax = max(1, min(U, 12))
                    k = int(rng.integers(1, kmax + 1))
                    while 256 * ((U + k - 1) // k) + (b - 256 * U) > 2 * MiB:
                        k += 1
                    nb[i], ks[i] = b, k
                    left -= b
            nb[0] = left
            so, do = int(rng.integers(0, 16)), int(rng.integers(0, 16))
            host = synth.payload(n, 700 + case)
            src = sbuf[so:so + n]
            src.copy_(torch.from_numpy(host))
            dview.fill_(0xA5)
            dst = base + CAN + do
            torch.cuda.synchronize()
            c0.send(src, n, 1, tag=case, cfg=c0.make_config(nb, ks, 0, 1))
            c1.recv(dst, n, 0, tag=case)
            W.run()
            got = dview.cpu().numpy()
            exp = np.zeros(n, dtype=np.uint8)
            X.replay(host, nb, ks, kinds, 256, exp)
            assert np.array_equal(got[CAN + do:CAN + do + n], exp), (case, n, nb, ks, so, do)
            assert (got[:CAN + do] == 0xA5).all() and (got[CAN + do + n:] == 0xA5).all(), ("canary", case)
            done += 1
        assert done == 24


def test_emulated_limits_refused(torch_cuda, monkeypatch):
    """The emulated world's own rule fails loudly, before any state changes: a 65th
    rendezvous receive of one pair recorded for the same run (every receive posts its
    clear-to-send at once) is MP_ERR_INVALID, and the 64 recorded messages still go
    through; mp_finalize on one of its contexts is MP_ERR_STATE."""
    torch = torch_cuda
    from paper_conf_sc_sojoodiasfga25_b200 import mp
    monkeypatch.setenv("MPX_EAGER", "0")
    with world(2, host_path=0) as W:
        c0, c1 = W.ctx[0], W.ctx[1]
        host, src = fill(torch, 8192, 1)
        dst = c1.alloc(65 * 8192)
        for m in range(64):
            c1.recv(dst + m * 8192, 8192, 0, tag=m)
            c0.send(src, 8192, 1, tag=m)
        with pytest.raises(mp.MPError) as e:
            c1.recv(dst + 64 * 8192, 8192, 0, tag=64)
        assert e.value.status == mp.MP_ERR_INVALID
        W.run()
        got = mp.as_tensor(dst, 64 * 8192).cpu().numpy().reshape(64, 8192)
        assert all(np.array_equal(g, host) for g in got)
        assert mp.lib().mp_finalize(c0.h) == mp.MP_ERR_STATE
