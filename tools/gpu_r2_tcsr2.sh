mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 300 python tools/tcsr_probe.py 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -k "tcsr or sample or dedup" 2>&1 | tail -2
REPS=2 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/tcsr_launches3.csv python tools/tcsr_probe.py > /dev/null 2>&1; echo ncu rc=$?
timeout 600 python -m pytest tests/test_gpu_cache.py -q -m gpu -p no:cacheprovider 2>&1 | tail -2
