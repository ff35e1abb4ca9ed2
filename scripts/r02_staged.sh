#!/bin/bash
# Staged-path efficiency check (round 2): loopback bench per_path, relay sweep, and the
# multi-rank per-path timing under MPS (all ranks on one GPU).  Usage: bash scripts/r02_staged.sh <tag>
TAG=${1:-r02}
PYT=${PYT:-1}
OUT=gpurun_out/$TAG
mkdir -p $OUT
[ "$PYT" = 1 ] && { timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo rc=$? >> $OUT/pytest_gpu.log; }
timeout 300 python bench.py --steps 200 --no-cpu-baseline > $OUT/bench.log 2>&1
timeout 300 python scripts/relay_sweep.py > $OUT/relay_sweep.jsonl 2>&1
for W in 3; do
  for N in 67108864 268435456; do
    MPX_BENCH_SAME_GPU=1 DIAG_BYTES=$N timeout 400 bash scripts/with_mps.sh python -m torch.distributed.run \
      --nnodes=1 --nproc-per-node $W --master-addr 127.0.0.1 --master-port 29533 scripts/diag_world_perf.py \
      > $OUT/world_perf_w${W}_n${N}.jsonl 2> $OUT/world_perf_w${W}_n${N}.err
  done
done
echo done
