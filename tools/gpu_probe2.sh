mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
TGL_KV=tma timeout 300 python tools/kv_timeline.py fp32 2>&1 | tail -20
TGL_KV=bin timeout 300 python tools/kv_timeline.py fp32 2>&1 | tail -20
PROBE_KV=tma PROBE_MASKS=0 TGL_KV=tma timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/probe_launches.csv python tools/kv_probe.py fp32 > /dev/null 2>&1
python tools/launches.py gpurun_out/probe_launches.csv 2 2>&1 | head -30
