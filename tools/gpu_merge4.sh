mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_cache.py -x -q -p no:cacheprovider > gpurun_out/pytest_cache.log 2>&1; echo "cache rc=$?" >> gpurun_out/pytest_cache.log
tail -3 gpurun_out/pytest_cache.log
grep -q "cache rc=0" gpurun_out/pytest_cache.log || exit 1
timeout 600 python bench.py --no-cpu-baseline --cache 4194304 > gpurun_out/bench_reddit_cache4m.log 2>&1
timeout 900 python bench.py --config MAG --no-cpu-baseline --cache 4194304 > gpurun_out/bench_mag_cache.log 2>&1
for f in bench_reddit_cache4m bench_mag_cache; do tail -1 gpurun_out/$f.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$f', d['value'], d['ms_per_step'], d['e2e']['value'], d['clocks'])" || tail -5 gpurun_out/$f.log; done
