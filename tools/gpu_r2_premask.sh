# kv_pre costs on the GDELT / REDDIT tail block (probe build, TGL_DEBUG_MASK)
mkdir -p gpurun_out
TGL_NVCC_EXTRA="-DTGL_PROBE" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for cfg in GDELT REDDIT; do
echo "== $cfg"
CFG=$cfg PROBE_KV=pre PROBE_SPLIT=1 PROBE_MASKS=0,2,4,64,6,66,70,71 timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -9
done
