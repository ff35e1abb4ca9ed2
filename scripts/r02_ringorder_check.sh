#!/bin/bash
# After the cross-stream ring order: every multi-rank GPU test, and osu_latency /
# osu_bw at 4 KiB - 4 MiB with two ranks on one GPU under MPS (eager path cost).
cd /root/repo || exit 1
mkdir -p gpurun_out/ro
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ro/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q tests/test_world.py -m gpu > gpurun_out/ro/world.log 2>&1; echo "world rc=$?"; tail -1 gpurun_out/ro/world.log
MPX_BENCH_SAME_GPU=1 timeout 900 bash scripts/with_mps.sh python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29631 scripts/omb_world.py --min-bytes 4096 --max-bytes 4194304 --windows 1,16 \
  --out gpurun_out/ro/omb.jsonl > gpurun_out/ro/omb.log 2>&1; echo "omb rc=$?"
grep '"latency"' gpurun_out/ro/omb.jsonl | head -12
