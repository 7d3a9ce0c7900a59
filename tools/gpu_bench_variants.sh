# bench.py K|V time (tail block) per compile variant and config
mkdir -p gpurun_out
for v in "$@"; do
  TGL_NVCC_EXTRA="$v" python paper_conf_asplos_wangm24_b200/build.py -f > gpurun_out/build_v.log 2>&1 || { echo "build failed: $v"; tail -20 gpurun_out/build_v.log; continue; }
  for c in ${CONFIGS:-REDDIT MAG}; do
    timeout 400 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bv.log 2>&1
    python -c "
import json,sys
d=json.loads(open('gpurun_out/bv.log').read().strip().splitlines()[-1]); r=d['roofline']
print(f'== {sys.argv[1] or \"default\"} {sys.argv[2]}: value {d[\"value\"]:.4g} step {d[\"ms_per_step\"]:.4f} ms kv {r[\"per_launch_ms\"]:.4f} ms frac {r[\"frac\"]:.3f}')
" "$v" "$c" || tail -3 gpurun_out/bv.log
  done
done
python paper_conf_asplos_wangm24_b200/build.py -f > /dev/null 2>&1
