# node-proj mode: kv_pre role counters + masks (probe build), ncu of the dense_pre kernels
O=gpurun_out/npprof; mkdir -p $O
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0,2,4,64,66,70,71 PROBE_PROF=1 PROBE_PROF_KV=pre timeout 300 python tools/kv_probe.py fp32 > $O/probe.log 2>&1
tail -10 $O/probe.log
python -c "import __graft_entry__ as g; g.build()" > $O/build2.log 2>&1 || { tail -30 $O/build2.log; exit 1; }
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0 timeout 900 ncu --set full --import-source on --clock-control none -k regex:dense_pre -c 4 -o $O/dense_pre_gdelt python tools/kv_probe.py fp32 > $O/ncu.log 2>&1
tail -3 $O/ncu.log
