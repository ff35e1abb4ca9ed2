cd /root/repo || exit 1
mkdir -p gpurun_out/bell2
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/noorder/libmpx.so', defines=['MPX_NO_RING_ORDER'])" > /dev/null 2>&1 || exit 1
for i in 1 2 3 4 5; do
  MPX_LIB=/tmp/noorder/libmpx.so timeout 300 python -m pytest -q -x tests/test_world.py -m gpu -k "doorbell_flow" > gpurun_out/bell2/without_$i.log 2>&1; echo "no order $i rc=$? $(tail -1 gpurun_out/bell2/without_$i.log)"
done
for i in 1 2 3 4 5; do
  timeout 300 python -m pytest -q -x tests/test_world.py -m gpu -k "doorbell_flow" > gpurun_out/bell2/with_$i.log 2>&1; echo "order $i rc=$? $(tail -1 gpurun_out/bell2/with_$i.log)"
done
