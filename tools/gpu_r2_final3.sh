# final state: smoke, full GPU suite, default bench line (+ cpu baseline), GDELT launch list
O=gpurun_out/final3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 2000 python -m pytest tests -q -m gpu -p no:cacheprovider --durations=8 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
( time timeout 900 python bench.py ) > $O/bench_default.log 2>&1
tail -2 $O/smoke.log; tail -14 $O/pytest_gpu.log; grep metric $O/bench_default.log | cut -c1-250
