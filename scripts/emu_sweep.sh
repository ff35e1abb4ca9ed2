#!/bin/bash
# Relay-alone rate of the multi-rank kernels in the emulated world (one cooperative
# grid) over ring geometry and lanes, beside the loopback relay ring (design experiment).
mkdir -p gpurun_out/emusweep
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "--lanes 16" "--lanes 32" "--lanes 16 --no-host" "--lanes 32 --no-host"; do
  echo "# $cfg" >> gpurun_out/emusweep/relay2.log
  timeout 120 python scripts/emu_perf.py --case relay --reps 5 $cfg 2>&1 | cut -c1-300 >> gpurun_out/emusweep/relay2.log
done
