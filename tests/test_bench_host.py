"""Host logic of bench.py that needs no GPU: the compact exhaustive sweep behind the
bench line's `e_sel` (the metric's "model-vs-sweep optimum error %")."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

MiB = 1 << 20


def test_esel_grid_covers_the_path_kinds_and_splits_exactly():
    n, npaths = 1 << 30, 8          # config 3: direct + 6 relays + host
    g = bench.esel_grid(n, npaths, npaths - 1)
    assert len(g) == len({(tuple(b), tuple(c)) for b, c in g}) >= 20
    assert ([n] + [0] * 7, [1] + [0] * 7) in g                       # direct alone
    for nb, ch in g:
        assert sum(nb) == n and nb[0] > 0 and ch[0] == 1              # Eq 3: shares sum to n
        for i in range(1, npaths):
            assert (nb[i] == 0) == (ch[i] == 0)                       # unused paths have k = 0
            if nb[i]:
                assert nb[i] % 256 == 0 and nb[i] // ch[i] <= 30 * MiB  # A-aligned, chunks fit a slot
    kinds = {tuple(i for i in range(1, npaths) if nb[i]) for nb, _ in g}
    assert (7,) in kinds and (1,) in kinds and tuple(range(1, 7)) in kinds and tuple(range(1, 8)) in kinds


def _json_lines(out):
    import json
    return [json.loads(x) for x in out.splitlines() if x.startswith("{")]


def test_reference_arm_contract_n1_and_torchrun_n2():
    """bench.py --impl reference (the CPU oracle as it stands, no GPU needed): one JSON
    line with the metric, impl "reference", W >= 3 warm-up steps and an e2e object; under
    torchrun at N = 2 only rank 0 prints, the other rank exits 0."""
    import socket
    import subprocess
    env = dict(os.environ, OMP_NUM_THREADS="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "1"], capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = _json_lines(out.stdout)
    assert len(lines) == 1
    d = lines[0]
    assert d["impl"] == "reference" and d["metric"] == bench.METRIC and d["n_gpus"] == 1 and d["warmup"] >= 3
    assert d["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                          "--master-addr", "127.0.0.1", "--master-port", str(port),
                          os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2", "--steps", "1",
                          "--warmup", "1"], capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = _json_lines(out.stdout)
    assert len(lines) == 1 and lines[0]["impl"] == "reference" and lines[0]["n_gpus"] == 2
