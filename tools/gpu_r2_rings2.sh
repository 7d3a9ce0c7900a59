# kv_pre ring sweep around 4 / 5 / 4 (GDELT, node projections)
O=gpurun_out/rings2; mkdir -p $O
run() {
  lbl=$1; fl=$2; shift 2
  TGL_NVCC_EXTRA="$fl" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $lbl failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4))" || tail -3 $O/b.log
}
run base ""
run A3W5R4 "-DTGL_KV_PRE_ASTAGES=3 -DTGL_KV_PRE_WSTAGES=5 -DTGL_KV_PRE_REUSE=4"
run A4W5R3 "-DTGL_KV_PRE_ASTAGES=4 -DTGL_KV_PRE_WSTAGES=5 -DTGL_KV_PRE_REUSE=3"
run A4W4R3 "-DTGL_KV_PRE_ASTAGES=4 -DTGL_KV_PRE_WSTAGES=4 -DTGL_KV_PRE_REUSE=3"
run base2 ""
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
