#!/bin/bash
# A/B: Step-1 band windows launched from a stream (product) vs replayed from a CUDA
# graph (-DMPX_GRAPH_WINDOWS), each against the sweep's own window timing.
cd /root/repo || exit 1
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/gw/libmpx.so', defines=['MPX_GRAPH_WINDOWS'])" > /dev/null 2>&1 || exit 1
for i in 1 2; do
  echo "== stream windows, run $i"; timeout 600 python scripts/diag/band_vs_window.py 2>&1 | grep MiB
  echo "== graph windows, run $i"; MPX_LIB=/tmp/gw/libmpx.so timeout 600 python scripts/diag/band_vs_window.py 2>&1 | grep MiB
done
