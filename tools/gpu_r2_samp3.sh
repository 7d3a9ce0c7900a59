# sampler knobs: queries per warp (TGL_SAMPLE_Q) x min CTAs per SM (TGL_SAMPLE_MINB), GDELT
O=gpurun_out/samp3; mkdir -p $O
run() {
  lbl=$1; fl=$2; shift 2
  TGL_NVCC_EXTRA="$fl" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $lbl failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); s=d['sampler']; print('$lbl', '%.4e'%d['value'], round(d['ms_per_step'],4), 'sampler ms', round(s['ms_per_step'],4))" || tail -3 $O/b.log
}
run base ""
run Q8B4 "-DTGL_SAMPLE_Q=8 -DTGL_SAMPLE_MINB=4"
run Q2B8 "-DTGL_SAMPLE_Q=2 -DTGL_SAMPLE_MINB=8"
run Q4B8 "-DTGL_SAMPLE_Q=4 -DTGL_SAMPLE_MINB=8"
run base2 ""
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
