mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -x -k "sample or pipeline" 2>&1 | tail -3
CFG=GDELT timeout 600 python tools/sample_probe.py 2>&1 | tail -4
CFG=GDELT timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sample --csv --log-file gpurun_out/sample_launches2.csv python tools/sample_probe.py > /dev/null 2>&1; echo ncu=$?
