mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention" -p no:cacheprovider > gpurun_out/pytest_attn.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_attn.log
tail -4 gpurun_out/pytest_attn.log
timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -20
timeout 300 python tools/kv_probe.py bf16 2>&1 | tail -20
