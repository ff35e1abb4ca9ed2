#!/bin/bash
# Reading C28 on one GPU: the wake probe test (time-sliced and under MPS) and the
# config-3 bench at N = 3 under MPS (MPX_BENCH_SAME_GPU=1).
cd /root/repo || exit 1
mkdir -p gpurun_out/wake
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/wake/build.log 2>&1 || { tail gpurun_out/wake/build.log; exit 1; }
timeout 600 python -m pytest -q -x tests/test_world.py -m gpu -k "wake" > gpurun_out/wake/test_wake.log 2>&1; echo "wake test rc=$?"
timeout 600 bash scripts/with_mps.sh python -m pytest -q -x tests/test_world.py -m gpu -k "wake" > gpurun_out/wake/test_wake_mps.log 2>&1; echo "wake mps rc=$?"
run3() {  # $1 = log name, $2 = ranks, rest = env
  local log=$1; local np=$2; shift 2
  env "$@" MPX_BENCH_SAME_GPU=1 MPX_WAKE_DEBUG=1 timeout 900 bash scripts/with_mps.sh python -X faulthandler -m torch.distributed.run \
    --nnodes=1 --nproc-per-node $np --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus $np --steps 5 --warmup 3 \
    > gpurun_out/wake/$log 2>&1
  echo "$log rc=$?"

}
run3 bench3_wake0.log 3 MPX_RELAY_WAKE_US=0
run3 bench3.log 3
run3 bench4.log 4
python scripts/bench_line_summary.py gpurun_out/wake/bench3_wake0.log gpurun_out/wake/bench3.log gpurun_out/wake/bench4.log
timeout 1500 python -m pytest -q tests/test_world.py tests/test_collectives.py -m gpu > gpurun_out/wake/test_world_all.log 2>&1; echo "world gpu tests rc=$?"; tail -3 gpurun_out/wake/test_world_all.log
