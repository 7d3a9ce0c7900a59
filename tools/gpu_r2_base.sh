# round-2 baseline: full GPU suite + GDELT bench (timed) as it stands
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
lscpu > gpurun_out/lscpu.txt; nproc >> gpurun_out/lscpu.txt
( time timeout 900 python bench.py --config GDELT --steps 20 --warmup 5 --no-cpu-baseline ) > gpurun_out/bench_gdelt.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log; tail -5 gpurun_out/bench_gdelt.log | cut -c1-600
