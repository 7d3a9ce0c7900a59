# wait-policy sweep for kv_pre on GDELT (node projections on): polling vs suspend, sleep lengths
O=gpurun_out/sleep; mkdir -p $O
run() {  # $1 label, $2 extra nvcc flags
  TGL_NVCC_EXTRA="$2" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $1 failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$1', round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4))" || tail -3 $O/b.log
}
run base ""
run suspend "-DTGL_PRE_SUSPEND"
run load512 "-DTGL_SLEEP_LOAD=512 -DTGL_SLEEP_W=256"
run epi512 "-DTGL_SLEEP_EPI=512 -DTGL_SLEEP_DESC=1024"
run all "-DTGL_SLEEP_LOAD=512 -DTGL_SLEEP_W=256 -DTGL_SLEEP_EPI=512 -DTGL_SLEEP_DESC=1024"
run base2 ""
