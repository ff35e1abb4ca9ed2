mkdir -p gpurun_out/trace
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python -c "from paper_conf_sc_sojoodiasfga25_b200 import _build as b; b.build(out='/tmp/trace/libmpx.so', defines=['MPX_TRACE'])" > gpurun_out/trace/build.log 2>&1
MPX_LIB=/tmp/trace/libmpx.so timeout 300 python scripts/diag/lane_trace.py > gpurun_out/trace/trace3.log 2>&1
for lanes in 16 32; do
  echo "# lanes $lanes" >> gpurun_out/trace/perf3.log
  timeout 120 python scripts/emu_perf.py --case relay --reps 5 --lanes $lanes --no-host 2>&1 | grep -o '"payload_GBps": [0-9.]*' >> gpurun_out/trace/perf3.log
done
timeout 300 python -m pytest tests/test_emulated_gpu.py -q -p no:cacheprovider -x > gpurun_out/trace/pytest3.log 2>&1; echo rc=$? >> gpurun_out/trace/pytest3.log
