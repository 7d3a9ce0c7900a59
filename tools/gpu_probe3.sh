mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention" -p no:cacheprovider 2>&1 | tail -2
PROBE_MASKS=0,2,95 timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -6
PROBE_MASKS=0 timeout 300 python tools/kv_probe.py bf16 2>&1 | tail -2
