# what bounds kv_pre / kv_pre2 on the GDELT tail block: debug masks (probe build)
# 2 skip gathers, 4 skip MMAs, 64 skip time warps, 1 skip epilogue math
mkdir -p gpurun_out
TGL_NVCC_EXTRA="-DTGL_PROBE" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for prec in fp32 bf16; do
echo "== GDELT $prec"
CFG=GDELT PROBE_KV=pre,pre2 PROBE_MASKS=0,1,2,4,64,6,66,70,71 timeout 600 python tools/kv_probe.py $prec 2>&1 | tail -19
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
