mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
PROBE_KV=async PROBE_MASKS=0 PROBE_TRACE=1 PROBE_TRACE_MASK=95 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/trace95.log 2>&1
PROBE_KV=async PROBE_MASKS=0 PROBE_TRACE=1 PROBE_TRACE_MASK=0 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/trace0.log 2>&1
PROBE_KV=async PROBE_MASKS=0,16,31,95,127,2047,4095 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/probe_masks.log 2>&1
tail -n 12 gpurun_out/probe_masks.log
