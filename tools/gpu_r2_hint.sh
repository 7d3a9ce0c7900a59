mkdir -p gpurun_out
run() { lbl=$1; shift
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/b.log 2>&1
  grep metric gpurun_out/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], d['config']['precision'], round(d['value']), round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4), 'frac', round(r['frac'],3))" || tail -3 gpurun_out/b.log
}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "attention_vs_oracle and pre" 2>&1 | tail -1
run hint --config GDELT
run hint --config GDELT --precision bf16
run hint --config REDDIT
run hint --config GDELT
