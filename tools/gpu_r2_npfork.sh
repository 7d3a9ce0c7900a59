# node_proj on a side stream overlapping the sampling launches
O=gpurun_out/fork; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_shard.py -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for i in 1 2; do
timeout 300 python bench.py --no-cpu-baseline > $O/bench_$i.log 2>&1
grep metric $O/bench_$i.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('GDELT', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'e2e %.3e'%d['e2e']['value'])" || tail -3 $O/bench_$i.log
done
