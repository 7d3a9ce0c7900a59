# kv_pre ring depths / weight reuse across tiles (node-projection GDELT + MAG)
O=gpurun_out/rings; mkdir -p $O
run() {  # $1 label, $2 extra nvcc flags, rest bench args
  lbl=$1; fl=$2; shift 2
  TGL_NVCC_EXTRA="$fl" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $lbl failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4))" || tail -3 $O/b.log
}
run base ""
run A5W4R3 "-DTGL_KV_PRE_ASTAGES=5 -DTGL_KV_PRE_WSTAGES=4 -DTGL_KV_PRE_REUSE=3"
run A4W5R4 "-DTGL_KV_PRE_ASTAGES=4 -DTGL_KV_PRE_WSTAGES=5 -DTGL_KV_PRE_REUSE=4"
run A6W3R2 "-DTGL_KV_PRE_ASTAGES=6 -DTGL_KV_PRE_WSTAGES=3 -DTGL_KV_PRE_REUSE=2"
run base2 ""
run A5W4R3 "-DTGL_KV_PRE_ASTAGES=5 -DTGL_KV_PRE_WSTAGES=4 -DTGL_KV_PRE_REUSE=3" --config MAG
run base "" --config MAG
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
