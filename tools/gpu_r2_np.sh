# node projections: parity tests, smoke, bench on/off (GDELT, REDDIT), kv probe
O=gpurun_out/np; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_nodeproj.py -x -q -p no:cacheprovider > $O/pytest_np.log 2>&1; echo "rc=$?" >> $O/pytest_np.log
tail -15 $O/pytest_np.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log; tail -2 $O/smoke.log
for np in on off; do for c in GDELT REDDIT; do
timeout 600 python bench.py --config $c --node-proj $np --no-cpu-baseline --no-e2e > $O/bench_${c}_$np.log 2>&1
grep metric $O/bench_${c}_$np.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c $np', round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), d.get('breakdown_ms_eager'))" || tail -5 $O/bench_${c}_$np.log
done; done
