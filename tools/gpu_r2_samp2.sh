mkdir -p gpurun_out
for v in "4 6"; do set -- $v
  TGL_NVCC_EXTRA="-DTGL_SAMPLE_Q=$1 -DTGL_SAMPLE_MINB=$2" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { echo "build $v failed"; tail -5 gpurun_out/build.log; continue; }
  echo "Q=$1 minB=$2"; timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -x -k "sample" 2>&1 | tail -1; CFG=GDELT timeout 600 python tools/sample_probe.py 2>&1 | grep flushed
done
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CFG=GDELT timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sample --csv --log-file gpurun_out/sample_launches3.csv python tools/sample_probe.py > /dev/null 2>&1; echo ncu=$?
