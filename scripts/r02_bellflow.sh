#!/bin/bash
# Many concurrent relayed messages (80 streams through one relay): the bell_flow
# scenario with the product library and with a variant built without the cross-stream
# ring order (MPX_NO_RING_ORDER); then every multi-rank GPU test.
cd /root/repo || exit 1
mkdir -p gpurun_out/bell
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/bell/build.log 2>&1 || exit 1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/noorder/libmpx.so', defines=['MPX_NO_RING_ORDER'])" >> gpurun_out/bell/build.log 2>&1 || exit 1
for i in 1 2 3; do
  timeout 600 python -m pytest -q -x tests/test_world.py -m gpu -k "doorbell_flow" > gpurun_out/bell/with_$i.log 2>&1; echo "ring order, run $i rc=$? $(tail -1 gpurun_out/bell/with_$i.log)"
done
MPX_LIB=/tmp/noorder/libmpx.so timeout 600 python -m pytest -q -x tests/test_world.py -m gpu -k "doorbell_flow" > gpurun_out/bell/without.log 2>&1; echo "without rc=$? $(tail -1 gpurun_out/bell/without.log)"
grep -h "rank .* failed\|Error" gpurun_out/bell/without.log | head -8
timeout 900 python -m pytest -q tests/test_world.py tests/test_collectives.py -m gpu > gpurun_out/bell/world.log 2>&1; echo "world rc=$?"; tail -2 gpurun_out/bell/world.log
