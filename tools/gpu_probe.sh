mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
PROBE_KV=async PROBE_PROF=1 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/probe_fp32.log 2>&1
PROBE_KV=async PROBE_MASKS=0,2,64,66 PROBE_WINDOW=0 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/probe_direct.log 2>&1
PROBE_KV=async PROBE_MASKS=0,2,64 PROBE_WINDOW=131072 timeout 300 python tools/kv_probe.py fp32 > gpurun_out/probe_w17.log 2>&1
PROBE_KV=async PROBE_MASKS=0,2,4,64 timeout 300 python tools/kv_probe.py bf16 > gpurun_out/probe_bf16.log 2>&1
PROBE_KV=async PROBE_MASKS=0 TGL_KV=async timeout 900 ncu --set full --import-source on --clock-control none -k regex:kv_async -s 2 -c 1 -o gpurun_out/kv_async python tools/kv_probe.py fp32 > gpurun_out/ncu_kv.log 2>&1
python tools/ncu_summary.py gpurun_out/kv_async.ncu-rep > gpurun_out/kv_async_summary.txt 2>&1
tail -n 12 gpurun_out/probe_*.log
