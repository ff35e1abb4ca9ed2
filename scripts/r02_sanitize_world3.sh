#!/bin/bash
# compute-sanitizer memcheck over the multi-rank tests (relay kernels with doorbell
# acknowledgements, gates, lingering relays, eager slots, the wake probe), every
# process.  Usage: bash scripts/r02_sanitize_world3.sh [all]
OUT=gpurun_out/r02/san3
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
SELS=("engine_same_gpu and 3" "relay_burst")
if [ "$1" = all ]; then SELS+=("doorbell_flow" "relay_wake" "eager_protocol and 3" "collectives and 3" "device_sync"); fi
for sel in "${SELS[@]}"; do
  tag=$(echo "$sel" | tr ' ' '_')
  MPX_TEST_SHOW_OUTPUT=1 MPX_TEST_STACKS_S=1400 timeout 1700 compute-sanitizer --tool memcheck --target-processes all --error-exitcode 99 --print-limit 50 \
    python -m pytest tests/test_world.py -q -s -p no:cacheprovider -m gpu -k "$sel" > $OUT/memcheck_$tag.log 2>&1
  echo "$sel rc=$?"; grep -h "ERROR SUMMARY\|passed\|failed" $OUT/memcheck_$tag.log | sort | uniq -c | head -5
done
