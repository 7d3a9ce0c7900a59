# GDELT ablations on the round-2 path: dedup / time precompute (SURVEY: "off / off (also run on)")
O=gpurun_out/abl; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
run() { lbl=$1; shift
  timeout 400 python bench.py --no-cpu-baseline "$@" > $O/bench_$lbl.log 2>&1
  grep metric $O/bench_$lbl.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), 'e2e %.3e'%d['e2e']['value'], {k: round(v,3) for k,v in d.get('breakdown_ms_eager').items()})" || tail -3 $O/bench_$lbl.log
}
run gdelt_dedup --dedup on
run gdelt_pre --precompute on
run gdelt_dedup_pre --dedup on --precompute on
run gdelt_dedup_pre_cache --dedup on --precompute on --cache 4194304
