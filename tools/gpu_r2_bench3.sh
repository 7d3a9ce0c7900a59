# bench lines: GDELT fp32 / bf16, REDDIT (+ prof variants of kv_pre ring depths)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "attention_vs_oracle and pre" > gpurun_out/pytest_pre.log 2>&1; tail -1 gpurun_out/pytest_pre.log
for args in "--config GDELT" "--config GDELT --precision bf16" "--config REDDIT"; do
  timeout 600 python bench.py $args --no-cpu-baseline --no-e2e > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$args', round(d['value']), round(d['ms_per_step'],4), round(r['per_launch_ms'],4), 'frac', round(r['frac'],3), 'pipe', round(r['tensor']['pipe_frac_bf16_peak'],3))" || tail -5 gpurun_out/b.log
done
for v in "6 3" "8 2" "5 4"; do set -- $v
  TGL_NVCC_EXTRA="-DTGL_KV_PRE_ASTAGES=$1 -DTGL_KV_PRE_WSTAGES=$2" python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "build $v failed"; continue; }
  timeout 600 python bench.py --config GDELT --no-cpu-baseline --no-e2e > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('A=$1 W=$2', round(d['value']), round(d['ms_per_step'],4), round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 gpurun_out/b.log
done
