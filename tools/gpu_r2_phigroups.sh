# group-mapped Phi (4 rows per thread) in kv_pre's time warps (-DTGL_PHI_GROUPS) vs the row-mapped default
O=gpurun_out/phigroups; mkdir -p $O
run() {  # $1 label, $2 extra nvcc flags, rest bench args
  lbl=$1; fl=$2; shift 2
  TGL_NVCC_EXTRA="$fl" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { echo "build $lbl failed"; tail -5 $O/build.log; return; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > $O/b.log 2>&1
  grep metric $O/b.log | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lbl', d['config']['workload'], '%.4e'%d['value'], round(d['ms_per_step'],4), 'kv', round(r['per_launch_ms'],4))" || tail -3 $O/b.log
}
TGL_NVCC_EXTRA="-DTGL_PHI_GROUPS" python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
TGL_NVCC_EXTRA="-DTGL_PHI_GROUPS" timeout 900 python -m pytest tests/test_gpu_nodeproj.py tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "node_proj or attention or pipeline or fused" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
run cols "-DTGL_PHI_GROUPS"
run base ""
run cols "-DTGL_PHI_GROUPS" --config MAG
run base "" --config MAG
run cols "-DTGL_PHI_GROUPS" --config REDDIT
run base "" --config REDDIT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
