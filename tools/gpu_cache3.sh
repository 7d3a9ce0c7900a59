mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_cache.py tests/test_abi_cpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_cache.log 2>&1; echo "cache rc=$?" >> gpurun_out/pytest_cache.log
tail -30 gpurun_out/pytest_cache.log
grep -q "cache rc=0" gpurun_out/pytest_cache.log || exit 1
timeout 600 python bench.py --no-cpu-baseline --cache 1048576 > gpurun_out/bench_cache.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_cache.csv python bench.py --steps 6 --warmup 3 --no-cpu-baseline --cache 1048576 > gpurun_out/bench_ncu_cache.log 2>&1
python tools/launches.py gpurun_out/launches_cache.csv > gpurun_out/step_share_cache.txt 2>&1
head -24 gpurun_out/step_share_cache.txt
tail -1 gpurun_out/bench_cache.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cache', d['value'], d['ms_per_step'], d['sampled_edges_per_s'], d['e2e']['value'], d['gpu_launches_per_step'])"
