#!/bin/bash
# Multi-rank harness on ONE GPU under MPS (all ranks share GPU 0): bench.py config 3 at
# N = 2, 3, 4, the config-2 sweep at N = 4, the OMB sweep at N = 3.  Functional runs
# of the multi-GPU paths, not NVLink numbers.  Usage: bash scripts/r02_world.sh <tag>
TAG=${1:-r02/world}
OUT=gpurun_out/$TAG
mkdir -p $OUT
export MPX_BENCH_SAME_GPU=1
run() {  # run <nproc> <port> <logname> <script + args>
  local np=$1 port=$2 name=$3; shift 3
  timeout ${TMO:-600} bash scripts/with_mps.sh python -m torch.distributed.run --nnodes=1 --nproc-per-node $np \
    --master-addr 127.0.0.1 --master-port $port "$@" > $OUT/$name.jsonl 2> $OUT/$name.err
  echo "$name rc=$?" >> $OUT/rc.txt
}
for N in 2 3 4; do
  run $N $((29600 + N)) bench_n$N bench.py --gpus $N --steps ${STEPS:-20} --warmup 3
done
TMO=900 run 4 29611 sweep_world scripts/sweep_world.py --sizes ${SWEEP_SIZES:-16,64} --step ${SWEEP_STEP:-16} --reps 3 --out $OUT/sweep_world.json
TMO=900 run 3 29612 omb_world scripts/omb_world.py --max-bytes ${OMB_MAX:-268435456} --windows 1,16 --out $OUT/omb_world_full.jsonl
echo done
