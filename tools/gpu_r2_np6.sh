# NP v6: FFN zo via TMEM init, 8-deep dense_pre weight ring; parity + benches on/off
O=gpurun_out/np6; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "node_proj or attention or pipeline or dense" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -4 $O/pytest.log
for c in GDELT REDDIT LASTFM WIKI; do for np in on off; do
timeout 300 python bench.py --config $c --node-proj $np --no-cpu-baseline --no-e2e > $O/bench_${c}_$np.log 2>&1
grep metric $O/bench_${c}_$np.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c $np', round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), {k: round(v,3) for k,v in d.get('breakdown_ms_eager').items()})" || tail -3 $O/bench_${c}_$np.log
done; done
