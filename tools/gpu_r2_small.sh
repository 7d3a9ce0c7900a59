# code-size experiment: kv_pre with rolled epilogue / Phi group loops (-DTGL_SMALL_CODE)
O=gpurun_out/small; mkdir -p $O
run() {  # $1 label, $2 extra nvcc flags, rest bench args
  lbl=$1; fl=$2; shift 2
  TGL_NVCC_EXTRA="$fl" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $lbl failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4))" || tail -3 $O/b.log
}
run base "" 
run small "-DTGL_SMALL_CODE"
run base "" --config REDDIT
run small "-DTGL_SMALL_CODE" --config REDDIT
run base "" --node-proj off
run small "-DTGL_SMALL_CODE" --node-proj off
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
