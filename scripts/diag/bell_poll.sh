#!/bin/bash
# Design experiment: how soon the emulated relay role sees a doorbell in pinned host
# memory, by the load that polls it (MPX_BELL_POLL 0 relaxed.sys, 1 volatile, 2 .cv,
# 3 relaxed.gpu), MPX_TRACE builds.
mkdir -p gpurun_out/bellpoll
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for m in 0 1 2 3; do
  python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/bp$m/libmpx.so', defines=['MPX_TRACE', 'MPX_BELL_POLL=$m'])" > gpurun_out/bellpoll/build$m.log 2>&1
  echo "# poll $m" >> gpurun_out/bellpoll/start.log
  MPX_LIB=/tmp/bp$m/libmpx.so timeout 200 python scripts/diag/lane_trace.py 2>&1 | grep -E "start path|last store" >> gpurun_out/bellpoll/start.log
done
