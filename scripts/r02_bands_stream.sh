#!/bin/bash
# C21 with stream-launched, spin-fronted windows and 1.5x band samples: the band model
# against the sweep's window timing, the band / osu_bw window GPU tests, and the
# loopback sweep (E_sel, E_pred).
cd /root/repo || exit 1
OUT=gpurun_out/bands2
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || exit 1
timeout 600 python scripts/diag/band_vs_window.py > $OUT/band_vs_window.txt 2>&1; head -14 $OUT/band_vs_window.txt
timeout 900 python -m pytest -q -s tests/test_engine_gpu.py -k "calibrate_bands or osu_bw_windows or window" > $OUT/tests.log 2>&1; echo "tests rc=$?"; grep -h "E_pred\|passed\|failed" $OUT/tests.log | tail -5
timeout 2400 python scripts/sweep.py --out $OUT/sweep.json > $OUT/sweep.log 2>&1; echo "sweep rc=$?"; grep -h "E_pred" $OUT/sweep.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print({k:(round(v,4) if isinstance(v,float) else v) for k,v in d.items() if 'E_' in k or k=='n'})"
