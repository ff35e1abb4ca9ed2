#!/usr/bin/env python3
"""One line per bench log: value, executed split, model prediction, E_pred, the pair
(0, 1)'s fitted β [GB/s] and relay wakes [µs] (reading C28).
    python scripts/bench_line_summary.py gpurun_out/wake/bench3.log ..."""
import json
import sys

for f in sys.argv[1:]:
    line = next((ln for ln in open(f, errors="replace") if ln.startswith('{"metric"')), None)
    if line is None:
        print(f, "no bench line")
        continue
    d = json.loads(line)
    m = d.get("model", {})
    prm = m.get("params", [])
    print(f, round(d["value"], 1), m.get("split"), "pred", round(m.get("predicted_GBps") or 0, 1),
          "E_pred", round(m.get("E_pred") or 0, 3), "beta", [round(p["beta"] / 1e9) for p in prm],
          "wake_us", [round(p.get("wake", 0) * 1e6, 1) for p in prm])
