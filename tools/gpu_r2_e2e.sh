# serving loop: H2D on the copy stream into a 2-deep landing buffer + one D2D
O=gpurun_out/e2e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "host or stream or staging or e2e" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
for c in GDELT REDDIT; do
timeout 400 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.log 2>&1
grep metric $O/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print('$c', '%.4e'%d['value'], 'e2e %.4e'%d['e2e']['value'], round(d['ms_per_step'],4))" || tail -3 $O/bench_$c.log
done
