# kv_pre default rings A4 / W5 / reuse 4: parity (all attention + pipeline cases) + benches
O=gpurun_out/ringdef; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_cache.py tests/test_gpu_host.py -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for c in GDELT REDDIT LASTFM WIKI MAG; do
timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e > $O/bench_$c.log 2>&1
grep metric $O/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 $O/bench_$c.log
done
timeout 300 python bench.py --node-proj off --no-cpu-baseline --no-e2e > $O/bench_noproj.log 2>&1
grep metric $O/bench_noproj.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('GDELT noproj', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))"
