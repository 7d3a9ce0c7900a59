# single-pass segmented walk in the bin epilogue
O=gpurun_out/np9; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "node_proj or attention or pipeline or time" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for c in GDELT REDDIT; do for np in auto off; do
timeout 300 python bench.py --config $c --node-proj $np --no-cpu-baseline --no-e2e > $O/bench_${c}_$np.log 2>&1
grep metric $O/bench_${c}_$np.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c $np', round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), {k: round(v,3) for k,v in d.get('breakdown_ms_eager').items()})" || tail -3 $O/bench_${c}_$np.log
done; done
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > $O/buildp.log 2>&1 || { tail -30 $O/buildp.log; exit 1; }
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0,1,64 PROBE_PROF=1 PROBE_PROF_KV=pre timeout 300 python tools/kv_probe.py fp32 > $O/probe.log 2>&1
tail -5 $O/probe.log
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
