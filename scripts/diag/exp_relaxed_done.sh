#!/bin/bash
# Emulated message times for the direct and the relay path at several sizes
# (completion-counting experiments).
mkdir -p gpurun_out/exprel
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for case in direct relay; do
  for mib in 16 64 256; do
    echo "# $case $mib MiB" >> gpurun_out/exprel/${OUTNAME:-run}.log
    timeout 120 python scripts/emu_perf.py --case $case --reps 9 --mib $mib --chunk-mib 4 2>&1 | grep -o '"s_median": [0-9.e-]*\|"payload_GBps": [0-9.]*' >> gpurun_out/exprel/${OUTNAME:-run}.log
  done
done
