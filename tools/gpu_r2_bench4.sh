# kv_pre wait flavours on GDELT fp32 / bf16
mkdir -p gpurun_out
for extra in "" "-DTGL_PRE_SUSPEND" "-DTGL_SLEEP_LOAD=256 -DTGL_SLEEP_DESC=512"; do
  TGL_NVCC_EXTRA="$extra" python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "build $extra failed"; continue; }
  for prec in fp32 bf16; do
  timeout 600 python bench.py --config GDELT --precision $prec --no-cpu-baseline --no-e2e > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('[$extra] $prec', round(d['value']), round(d['ms_per_step'],4), round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 gpurun_out/b.log
  done
done
