#!/bin/bash
# Round-2 GPU session: tests, bench (both arms), ncu launch list + full captures of the
# top kernels, the emulated multi-rank world, per-rank NVLink ncu pass (only on a box
# with >= 2 GPUs), loopback sweep.
# Usage (under gpurun): bash scripts/r02_profile.sh <tag>
TAG=${1:-r02/prof}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi -q -d CLOCK > $OUT/clocks_before.txt 2>&1
(nproc; grep -m1 "model name" /proc/cpuinfo) > $OUT/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "rc=$?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py --save-params $OUT/params.txt > $OUT/bench.log 2>&1; echo "rc=$?" >> $OUT/bench.log
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > $OUT/bench_reference.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"direct_kernel" -s 3 -c 1 -o $OUT/direct_full \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_direct.log 2>&1
RELAY_K=32 timeout 600 ncu --set full --clock-control none --import-source on -k regex:xfer_kernel -s 2 -c 1 \
  -o $OUT/relay_full python scripts/relay_one.py > $OUT/ncu_relay.log 2>&1
# multi-rank engine on one GPU: the emulated world (one cooperative grid over every rank)
timeout 900 python -m pytest tests/test_emulated_gpu.py -q -p no:cacheprovider > $OUT/pytest_emulated.log 2>&1
timeout 300 python scripts/emu_perf.py --mib 256 --out $OUT/emu_perf_256.jsonl > $OUT/emu_perf.log 2>&1
NG=$(nvidia-smi -L | wc -l)
if [ "$NG" -ge 2 ]; then  # per-rank NVLink counters need one GPU per rank (ncu serialises a shared device)
  NCU_OUT=$OUT/ncu_world timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $NG \
    --master-addr 127.0.0.1 --master-port 29650 --no-python scripts/ncu_rank.sh bench.py --gpus $NG --steps 5 \
    --warmup 3 > $OUT/ncu_world_bench.jsonl 2> $OUT/ncu_world_bench.err; echo "ncu_world rc=$?" >> $OUT/ncu_world_bench.err
  python scripts/nvlink_summary.py $OUT/ncu_world $NG 1073741824 --out profiles/ncu_nvlink.json > $OUT/nvlink_summary.json
fi
timeout 900 python scripts/sweep.py --out $OUT/sweep.json > $OUT/sweep.log 2>&1; echo "rc=$?" >> $OUT/sweep.log
nvidia-smi -q -d CLOCK > $OUT/clocks_after.txt 2>&1
echo done
