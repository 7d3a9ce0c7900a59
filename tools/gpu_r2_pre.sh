# kv_pre bring-up: unit + pipeline parity, then GDELT / REDDIT bench lines
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "split_rows or attention_vs_oracle or layouts" > gpurun_out/pytest_pre.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_pre.log
tail -3 gpurun_out/pytest_pre.log
grep -q "rc=0" gpurun_out/pytest_pre.log || { grep -B5 -A25 "Error\|assert" gpurun_out/pytest_pre.log | head -80; exit 1; }
timeout 600 python bench.py --config GDELT --no-cpu-baseline --steps 20 > gpurun_out/bench_gdelt_pre.log 2>&1; echo "rc=$?" >> gpurun_out/bench_gdelt_pre.log
timeout 600 python bench.py --config REDDIT --no-cpu-baseline > gpurun_out/bench_reddit_pre.log 2>&1
timeout 600 python bench.py --config GDELT --no-cpu-baseline --precision bf16 --no-e2e > gpurun_out/bench_gdelt_pre_bf16.log 2>&1
for f in bench_gdelt_pre bench_reddit_pre bench_gdelt_pre_bf16; do tail -1 gpurun_out/$f.log | python -c "
import json,sys
try:
  d=json.loads(sys.stdin.read()); r=d['roofline']; print('$f', round(d['value']), round(d['ms_per_step'],4), r['kernel'][:30], round(r['per_launch_ms'],4), round(r['frac'],3), d['breakdown_ms_eager'])
except Exception as e: print('$f failed', e)
"; done
tail -5 gpurun_out/bench_gdelt_pre.log | cut -c1-300
