mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_cache.py tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "cache or pipeline" > gpurun_out/pytest_cache.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_cache.log
tail -3 gpurun_out/pytest_cache.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log; tail -2 gpurun_out/smoke.log
