#!/bin/bash
# Short GPU session: smoke, every gpu test, bench (+ reference arm), the ncu launch list
# of the bench command and one full ncu capture of the benchmarked kernel.
# Usage (under gpurun): bash scripts/gpu_profile_short.sh <tag>
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
(nproc; grep -m1 "model name" /proc/cpuinfo) > $OUT/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "rc=$?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py --save-params $OUT/params.txt > $OUT/bench.log 2>&1; echo "rc=$?" >> $OUT/bench.log
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > $OUT/bench_reference.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"xfer_kernel|direct_kernel" -s 3 -c 1 -o $OUT/prof \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_full.log 2>&1
[ -f $OUT/prof.ncu-rep ] && ncu -i $OUT/prof.ncu-rep --page raw --csv > $OUT/prof_raw.csv 2>/dev/null
echo done
