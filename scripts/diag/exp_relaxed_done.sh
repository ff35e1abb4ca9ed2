#!/bin/bash
# Emulated direct-path message time at 16 / 256 MiB (completion counting experiments).
mkdir -p gpurun_out/exprel
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for mib in 16 64 256; do
  echo "# $mib MiB" >> gpurun_out/exprel/direct2.log
  timeout 120 python scripts/emu_perf.py --case direct --reps 9 --mib $mib 2>&1 | grep -o '"s_median": [0-9.e-]*\|"payload_GBps": [0-9.]*' >> gpurun_out/exprel/direct2.log
done
