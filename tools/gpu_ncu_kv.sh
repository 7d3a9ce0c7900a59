mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
PROBE_WINDOW=65536 PROBE_KV=tma PROBE_MASKS=0 TGL_KV=tma timeout 900 ncu --set full --import-source on --clock-control none -k regex:kv_tma -s 2 -c 1 -o gpurun_out/kv_tma python tools/kv_probe.py fp32 > gpurun_out/ncu_kv.log 2>&1
tail -3 gpurun_out/ncu_kv.log
ls -la gpurun_out
