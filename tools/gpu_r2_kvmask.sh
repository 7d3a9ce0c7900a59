# kv_split skeleton costs on the GDELT tail block (probe build, TGL_DEBUG_MASK)
mkdir -p gpurun_out
TGL_NVCC_EXTRA="-DTGL_PROBE" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
CFG=GDELT PROBE_KV=split PROBE_MASKS=0,64,1,16,65,14,78,79,95 timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -10
