#!/bin/bash
# Design experiment: Step 1's band windows behind a busy vs a sleeping spin kernel —
# the banded model's 64 KiB - 2 MiB prediction against spin-fronted windows.
mkdir -p gpurun_out/spin
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/sleep/libmpx.so', defines=['MPX_SPIN_SLEEP'])" > /dev/null 2>&1
for i in 1 2 3; do
  echo "# busy $i" >> gpurun_out/spin/ab.log; timeout 200 python scripts/diag/band64k.py 2>&1 | grep KiB >> gpurun_out/spin/ab.log
  echo "# sleep $i" >> gpurun_out/spin/ab.log; MPX_LIB=/tmp/sleep/libmpx.so timeout 200 python scripts/diag/band64k.py 2>&1 | grep KiB >> gpurun_out/spin/ab.log
done
