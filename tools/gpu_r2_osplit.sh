# FFN writes the split16 operand rows of the layer above (no split launch)
O=gpurun_out/osplit; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_host.py tests/test_gpu_cache.py tests/test_gpu_backward.py -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for c in GDELT REDDIT LASTFM; do
timeout 300 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.log 2>&1
grep metric $O/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'e2e %.3e'%d['e2e']['value'], d['gpu_launches_per_step'])" || tail -3 $O/bench_$c.log
done
