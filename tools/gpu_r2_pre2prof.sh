# per-role cycle counters of kv_pre2 vs kv_pre on the GDELT tail block (probe build)
mkdir -p gpurun_out
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for kv in pre pre2; do
  echo "== GDELT fp32 $kv"
  CFG=GDELT PROBE_KV=$kv PROBE_MASKS=0,2,4,64,71 PROBE_PROF=1 PROBE_PROF_KV=$kv timeout 300 python tools/kv_probe.py fp32 2>&1 | tail -8
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
