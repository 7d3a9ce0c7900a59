# round-2 iteration: build, changed GPU tests, GDELT + REDDIT bench lines
mkdir -p gpurun_out
free -g > gpurun_out/free.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_shard.py tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "shard or attention" > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
timeout 900 python bench.py --config GDELT > gpurun_out/bench_gdelt.log 2>&1; echo "rc=$?" >> gpurun_out/bench_gdelt.log
timeout 600 python bench.py --config REDDIT --no-cpu-baseline > gpurun_out/bench_reddit.log 2>&1
tail -5 gpurun_out/pytest_iter.log; tail -3 gpurun_out/bench_gdelt.log | cut -c1-400; tail -2 gpurun_out/bench_reddit.log | cut -c1-300
