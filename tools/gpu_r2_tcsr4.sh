# T-CSR one-sweep scatter staged through shared memory (coalesced runs): bit-exactness + time
O=gpurun_out/tcsr4; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_big.py -x -q -p no:cacheprovider -k "tcsr or full_config or gdelt_full" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
timeout 300 python tools/tcsr_probe.py 2>&1 | tail -2
timeout 400 python bench.py --no-cpu-baseline --no-e2e > $O/bench.log 2>&1; grep metric $O/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['tcsr'], '%.4e'%d['value'])"
