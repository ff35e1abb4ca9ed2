#!/bin/bash
# compute-sanitizer pass over the engine's GPU tests (memcheck, racecheck, synccheck).
# Usage (under gpurun): bash scripts/sanitize.sh <tag>
TAG=${1:-san}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
SEL="direct_only or single_staged_path or all_paths_misaligned or ragged_tail or send_recv_loopback or model_selected_transfer"
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 50 \
    python -m pytest tests/test_engine_gpu.py -q -p no:cacheprovider -k "$SEL" > $OUT/$tool.log 2>&1
  echo "rc=$?" >> $OUT/$tool.log
done
echo done
