#!/bin/bash
# Run one tests/_world_worker.py scenario with per-rank logs (diagnostics).
#   bash scripts/run_world_logs.sh <world> <scenario> <outdir> [timeout_s]
W=$1; SCEN=$2; OUT=$3; TO=${4:-200}
mkdir -p "$OUT"
PORT=$((20000 + RANDOM % 20000))
pids=()
for ((r = 0; r < W; r++)); do
  timeout "$TO" python tests/_world_worker.py $r $W $PORT $SCEN > "$OUT/rank$r.log" 2>&1 &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; echo "pid $p exit $?"; done
