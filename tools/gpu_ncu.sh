mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
PROBE_KV=async PROBE_MASKS=0 TGL_KV=async timeout 900 ncu --set full --import-source on --clock-control none -k regex:${KREGEX:-kv_async} -s 2 -c 1 -o gpurun_out/${NCU_OUT:-kv_async} python tools/kv_probe.py ${PREC:-fp32} > gpurun_out/ncu_kv.log 2>&1
tail -2 gpurun_out/ncu_kv.log
