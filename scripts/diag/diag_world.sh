#!/bin/bash
# Diagnose the multi-rank engine (one GPU per rank: tests/_world_worker.py puts rank r on GPU r).
# Usage: bash scripts/diag/diag_world.sh <outdir> <world> [MPX_NO_RELAY=0|1]
OUT=${1:-gpurun_out/diag}; W=${2:-3}; NR=${3:-0}
mkdir -p $OUT
PORT=$((20000 + RANDOM % 20000))
pids=()
for ((r=0; r<W; r++)); do
  MPX_DEBUG=1 MPX_NO_RELAY=$NR timeout 100 python tests/_world_worker.py $r $W $PORT engine > $OUT/w${W}_nr${NR}_rank$r.log 2>&1 &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; echo "pid $p rc=$?" >> $OUT/w${W}_nr${NR}_rc.txt; done
nvidia-smi --query-compute-apps=pid,used_memory --format=csv >> $OUT/w${W}_nr${NR}_rc.txt 2>&1
