#!/bin/bash
mkdir -p gpurun_out/trace
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/trace/libmpx.so', defines=['MPX_TRACE'])" > gpurun_out/trace/build.log 2>&1
MPX_LIB=/tmp/trace/libmpx.so timeout 300 python scripts/diag/direct_trace.py > gpurun_out/trace/direct.log 2>&1
