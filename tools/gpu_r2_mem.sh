# N3 memory parity, then the full GPU suite + smoke
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_memory.py -q -m gpu -p no:cacheprovider > gpurun_out/pytest_mem.log 2>&1; echo "mem rc=$?" >> gpurun_out/pytest_mem.log
tail -25 gpurun_out/pytest_mem.log
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider --durations=25 > gpurun_out/pytest_gpu_full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_full.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -35 gpurun_out/pytest_gpu_full.log; tail -2 gpurun_out/smoke.log
