mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 300 python tools/tcsr_probe.py 2>&1 | tail -1
timeout 600 python -m pytest tests/test_gpu_cache.py -q -m gpu -p no:cacheprovider 2>&1 | tail -2
TGL_NVCC_EXTRA="-DTGL_SW_NOLOOKBACK" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
echo "no lookback:"; timeout 300 python tools/tcsr_probe.py 2>&1 | tail -1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
