"""Multi-rank paths: world_size-2/3 process groups over gloo on 127.0.0.1.

CPU: the bootstrap all-gather and the per-pair model selection are consistent
across ranks.  GPU: the real multi-rank engine (IPC-mapped heaps, on-demand relay
kernels, shared pinned host ring), rank r on GPU r,
bit-exact against the oracle's reference transfer; one GPU per rank (need_gpus)."""
import os
import socket
import subprocess
import sys

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def run_world(world, scenario, timeout, env=None):
    port = free_port()
    penv = dict(os.environ, **(env or {}))
    procs = [subprocess.Popen([sys.executable, os.path.join(HERE, "_world_worker.py"), str(r), str(world),
                               str(port), scenario], stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True,
                              env=penv)
             for r in range(world)]
    outs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=timeout)
            outs.append(out)
    except subprocess.TimeoutExpired:
        for p in procs:
            if p.poll() is None:
                p.kill()
        tails = [p.communicate()[0][-2000:] for p in procs]
        raise AssertionError("timed out; per-rank output tails:\n" +
                             "\n".join(f"--- rank {r}\n{t}" for r, t in enumerate(tails)))
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    if os.environ.get("MPX_TEST_SHOW_OUTPUT") == "1":  # e.g. each rank's compute-sanitizer summary
        for r, out in enumerate(outs):
            print(f"--- rank {r} output tail\n{out[-1500:]}")
    bad = [(r, p.returncode, out) for r, (p, out) in enumerate(zip(procs, outs)) if p.returncode != 0]
    assert not bad, "\n".join(f"rank {r} failed (rc {rc}):\n{out[:2000]}\n...\n{out[-2000:]}" for r, rc, out in bad)


def need_gpus(world):
    """A multi-rank GPU test runs with one GPU per rank.  Ranks whose kernels wait on one
    another are never separate launches sharing a GPU (B200 profiling guide: nothing
    guarantees they run at the same time; processes spinning on one another raised
    Xid 109 there).  With fewer GPUs the same engine runs as an emulated world —
    one cooperative grid over every rank's kernels: tests/test_emulated_gpu.py."""
    torch = pytest.importorskip("torch")
    n = torch.cuda.device_count() if torch.cuda.is_available() else 0
    if n < world:
        pytest.skip(f"needs {world} GPUs (one per rank), found {n}; one-GPU coverage: test_emulated_gpu.py")


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_bootstrap_and_consistent_selection(world):
    run_world(world, "gloo_model", timeout=240)


@pytest.mark.parametrize("world", [2, 3, 4])
def test_bench_config3_roles_and_plan(world):
    # bench.py --gpus N: rank roles and the shared config-3 plan, gloo on CPU
    run_world(world, "bench_plan", timeout=240)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_multirank_engine(world):
    need_gpus(world)
    run_world(world, "engine", timeout=400)


@pytest.mark.gpu
def test_multirank_faults_reported_not_hung():
    need_gpus(2)
    run_world(2, "faults", timeout=300)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_multirank_registered_buffers(world):
    need_gpus(world)
    run_world(world, "register", timeout=400)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3, 4])
def test_multirank_collectives(world):
    # NEXT f3: mp_alltoall / mp_allreduce through the multi-rank engine
    need_gpus(world)
    run_world(world, "coll", timeout=600)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_multirank_eager_protocol(world):
    # reading C23: small messages skip the rendezvous
    need_gpus(world)
    run_world(world, "eager", timeout=400)


@pytest.mark.gpu
def test_multirank_device_sync_with_relays():
    # relay kernels are bounded launches (doorbell thread), so
    # torch.cuda.synchronize() between messages and during a relayed message is safe
    need_gpus(3)
    run_world(3, "devsync", timeout=400)


@pytest.mark.gpu
def test_multirank_engine_shallow_staged_pipelines():
    # every staged launch at 4 stages (MPX_STAGES=4): the send / recv / relay kernel
    # instances a sender with many relays gets (the default picks 6 when room allows)
    need_gpus(3)
    run_world(3, "engine", timeout=400, env={"MPX_STAGES": "4"})


@pytest.mark.gpu
def test_multirank_relay_burst_doorbell_wrap_and_linger():
    # 160 relayed messages: doorbell / decision rings wrap, lingering relay kernels
    # switch between streamed and per-chunk lanes, relaunch after quiet periods
    need_gpus(3)
    run_world(3, "relay_burst", timeout=400)


@pytest.mark.gpu
def test_multirank_config3_full_size_bit_exact():
    # BASELINE.json config 3 (1 GiB + 4099 B) through the multi-rank engine in the bench's
    # launch configuration: B200 pick, paper pick, every path at once; world 3
    need_gpus(3)
    run_world(3, "full_size", timeout=600)


@pytest.mark.gpu
def test_multirank_relay_wake_calibration():
    # reading C28: the collective wake probe after Step 1, the env override, and
    # relayed messages after it (world 3)
    need_gpus(3)
    run_world(3, "wake", timeout=400)


@pytest.mark.gpu
def test_multirank_doorbell_flow_control():
    # 112 relayed messages in flight through one relay (two receivers, 112 streams,
    # receives posted last-first): doorbell flow control and cross-stream ring order
    need_gpus(4)
    run_world(4, "bell_flow", timeout=500)
