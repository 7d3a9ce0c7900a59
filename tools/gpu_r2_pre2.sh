# kv_pre2 ring variants vs kv_pre on GDELT / REDDIT (fp32, bf16)
mkdir -p gpurun_out
run() {  # $1 label, rest bench args
  lbl=$1; shift
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], d['config']['precision'], round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 gpurun_out/b.log
}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run pre --config GDELT --kv-kernel pre
run pre2 --config GDELT --kv-kernel pre2
run pre2 --config GDELT --kv-kernel pre2 --precision bf16
run pre --config GDELT --kv-kernel pre --precision bf16
run pre2 --config REDDIT --kv-kernel pre2
for v in "6 6" "7 6" "8 2"; do set -- $v
  TGL_NVCC_EXTRA="-DTGL_KV_PRE2_ASTAGES=$1 -DTGL_KV_PRE2_WSTAGES=$2" python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "build $v failed"; continue; }
  run "pre2 A=$1 W=$2" --config GDELT --kv-kernel pre2
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
