# where the time warps' time goes (probe build): compute vs fence vs non-time passes
O=gpurun_out/tprof; mkdir -p $O
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > $O/buildp.log 2>&1 || { tail -30 $O/buildp.log; exit 1; }
for c in GDELT MAG; do
CFG=$c PROBE_KV=pre PROBE_MASKS=0 PROBE_PROF=1 PROBE_PROF_KV=pre timeout 600 python tools/kv_probe.py fp32 > $O/probe_$c.log 2>&1
tail -2 $O/probe_$c.log
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
