# per-role cycle counters of kv_pre (probe build) on the GDELT / REDDIT tail blocks
mkdir -p gpurun_out
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for cfg in GDELT REDDIT; do for prec in fp32 bf16; do
  echo "== $cfg $prec"
  CFG=$cfg PROBE_KV=pre PROBE_MASKS=0 PROBE_PROF=1 PROBE_PROF_KV=pre timeout 300 python tools/kv_probe.py $prec 2>&1 | tail -2
done; done
