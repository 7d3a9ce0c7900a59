# no-clobber stage stores + vectorised omega / phi loads in kv_pre's time warps: parity, benches, role counters
O=gpurun_out/v5; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "node_proj or attention or pipeline or fused" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for c in GDELT MAG REDDIT LASTFM; do
timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e > $O/bench_$c.log 2>&1
grep metric $O/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 $O/bench_$c.log
done
timeout 300 python bench.py --node-proj off --no-cpu-baseline --no-e2e > $O/bench_noproj.log 2>&1
grep metric $O/bench_noproj.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('GDELT noproj', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))"
TGL_NVCC_EXTRA="-DTGL_PROBE -DTGL_KV_PROF" python -c "import __graft_entry__ as g; g.build()" > $O/buildp.log 2>&1
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0 PROBE_PROF=1 PROBE_PROF_KV=pre timeout 600 python tools/kv_probe.py fp32 > $O/probe.log 2>&1; tail -1 $O/probe.log | cut -c1-400
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
