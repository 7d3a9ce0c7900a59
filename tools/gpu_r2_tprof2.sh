# time warps: with / without the cosine (mask 128), constant Phi (mask 256), no Phi (64)
O=gpurun_out/tprof2; mkdir -p $O
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > $O/buildp.log 2>&1 || { tail -30 $O/buildp.log; exit 1; }
for m in 0 128 256 64; do
CFG=GDELT PROBE_KV=pre PROBE_MASKS=$m PROBE_PROF=1 PROBE_PROF_KV=pre PROBE_PROF_MASK=$m timeout 600 python tools/kv_probe.py fp32 > $O/probe_$m.log 2>&1
echo "mask $m"; tail -2 $O/probe_$m.log | cut -c1-400
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
