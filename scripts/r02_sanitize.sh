#!/bin/bash
# Round-2 compute-sanitizer pass over the streamed-lane engine (memcheck, synccheck) and
# the multi-rank engine at world 2 (memcheck, all processes), plus two repeats of the
# GPU suite (flakiness check).  Usage (under gpurun): bash scripts/r02_sanitize.sh <tag>
TAG=${1:-r02/san}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
SEL="direct_only or single_staged_path or all_paths_misaligned or ragged_tail or send_recv_loopback or model_selected_transfer or staged_slices or two_streams"
for tool in memcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 50 \
    python -m pytest tests/test_engine_gpu.py -q -p no:cacheprovider -k "$SEL" > $OUT/$tool.log 2>&1
  echo "rc=$?" >> $OUT/$tool.log
done
timeout 1500 compute-sanitizer --tool memcheck --target-processes all --error-exitcode 99 --print-limit 50 \
  python -m pytest tests/test_world.py -q -p no:cacheprovider -k "engine_same_gpu and 2" > $OUT/memcheck_world.log 2>&1
echo "rc=$?" >> $OUT/memcheck_world.log
for i in 1 2; do
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_rep$i.log 2>&1
  echo "rc=$?" >> $OUT/pytest_gpu_rep$i.log
done
echo done
