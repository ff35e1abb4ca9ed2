cd /root/repo || exit 1
OUT=gpurun_out/r02/final2
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
timeout 600 python bench.py > $OUT/bench.log 2>&1; echo "bench rc=$?"; grep '"metric"' $OUT/bench.log | head -c 1500; echo
