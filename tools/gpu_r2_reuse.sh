mkdir -p gpurun_out
run() { lbl=$1; shift
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], d['config']['precision'], round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 gpurun_out/b.log
}
for v in "2 3 7" "0 3 7" "0 4 5" "1 3 7" "0 2 8"; do set -- $v
  TGL_NVCC_EXTRA="-DTGL_KV_PRE_REUSE=$1 -DTGL_KV_PRE_WSTAGES=$2 -DTGL_KV_PRE_ASTAGES=$3" python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "build $v failed"; continue; }
  run "R=$1 W=$2 A=$3" --config GDELT
  run "R=$1 W=$2 A=$3" --config GDELT --precision bf16
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
