#!/bin/bash
# One GPU session: smoke, gpu tests, bench, sweep, OMB sweeps (bw/bibw/latency, windows), small-message sweep,
# ncu launch list + per-path counters + one full capture.
# Usage (under gpurun): bash scripts/gpu_profile.sh <tag>
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi -q -d CLOCK > $OUT/clocks_before.txt 2>&1
(nproc; grep -m1 "model name" /proc/cpuinfo) > $OUT/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
# tools (not the product): C OMB harness and the copy design sweeps
[ -x scripts/omb_c ] || g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include scripts/omb_c.cpp \
  -L paper_conf_sc_sojoodiasfga25_b200/_lib -lmpx -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,'$ORIGIN/../paper_conf_sc_sojoodiasfga25_b200/_lib' -o scripts/omb_c
[ -x scripts/omb_window ] || g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include scripts/omb_window.cpp \
  -L paper_conf_sc_sojoodiasfga25_b200/_lib -lmpx -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,'$ORIGIN/../paper_conf_sc_sojoodiasfga25_b200/_lib' -o scripts/omb_window
[ -x scripts/smallbench ] || nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o scripts/smallbench scripts/smallbench.cu
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "rc=$?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py --save-params $OUT/params.txt > $OUT/bench.log 2>&1; echo "rc=$?" >> $OUT/bench.log
MPX_COPY=reg timeout 300 python bench.py --no-cpu-baseline --steps 200 --params $OUT/params.txt > $OUT/bench_reg.log 2>&1
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > $OUT/bench_reference.log 2>&1
timeout 900 python scripts/sweep.py --out $OUT/sweep.json > $OUT/sweep.log 2>&1; echo "rc=$?" >> $OUT/sweep.log
timeout 900 python scripts/omb.py --out $OUT/omb.jsonl > $OUT/omb.log 2>&1
timeout 900 ./scripts/omb_c > $OUT/omb_c.jsonl 2> $OUT/omb_c.err
timeout 900 ./scripts/omb_window bands > $OUT/omb_window_bands.jsonl 2> $OUT/omb_window.err
[ -x scripts/smallbench ] && timeout 300 ./scripts/smallbench > $OUT/smallbench.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_launch_bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum \
  --clock-control none --csv --log-file $OUT/path_probe.csv python scripts/path_probe.py > $OUT/path_probe.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"xfer_kernel|direct_kernel" -s 3 -c 1 -o $OUT/prof \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --params $OUT/params.txt > $OUT/ncu_full.log 2>&1
echo done
