mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention or time_encode" -p no:cacheprovider 2>&1 | tail -3
for w in 0 65536; do echo "window $w"; PROBE_WINDOW=$w PROBE_MASKS=0,2,6,95 timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -8; done
echo "window 2^22"; PROBE_MASKS=0,2 timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -4
PROBE_WINDOW=65536 PROBE_MASKS=0,2,6 timeout 300 python tools/kv_probe.py bf16 2>&1 | tail -6
PROBE_WINDOW=65536 TGL_KV=tma timeout 300 python tools/kv_timeline.py fp32 2>&1 | tail -20
