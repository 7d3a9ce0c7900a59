# iteration: build, targeted + full GPU tests, bench, launch list
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests -x -q -m gpu -p no:cacheprovider -k "dedup or sample" > gpurun_out/pytest_focus.log 2>&1; echo "focus rc=$?" >> gpurun_out/pytest_focus.log
tail -3 gpurun_out/pytest_focus.log
grep -q "focus rc=0" gpurun_out/pytest_focus.log || exit 1
timeout 1200 python -m pytest tests -x -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_fp32.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1
python tools/launches.py gpurun_out/launches.csv > gpurun_out/step_share.txt 2>&1
tail -2 gpurun_out/pytest_gpu.log; head -14 gpurun_out/step_share.txt; tail -1 gpurun_out/bench_fp32.log | cut -c1-400
