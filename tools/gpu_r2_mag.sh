# MAG on a split16-only node table (kv_pre + dense_pre), full-size parity + bench
O=gpurun_out/mag; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_big.py -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -5 $O/pytest.log
timeout 900 python bench.py --config MAG --no-cpu-baseline > $O/bench_MAG.log 2>&1
grep metric $O/bench_MAG.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('MAG', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), 'e2e %.3e'%d['e2e']['value'], r['kernel'][:40], d['tcsr']['build_ms'])" || tail -5 $O/bench_MAG.log
timeout 600 python bench.py --no-cpu-baseline --no-e2e > $O/bench_GDELT.log 2>&1
grep metric $O/bench_GDELT.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('GDELT', '%.4e'%d['value'], d['tcsr'])" || tail -3 $O/bench_GDELT.log
