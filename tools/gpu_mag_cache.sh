mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python bench.py --config MAG --no-cpu-baseline --dedup on > gpurun_out/bench_mag_dedup.log 2>&1
timeout 900 python bench.py --config MAG --no-cpu-baseline --cache 4194304 > gpurun_out/bench_mag_cache.log 2>&1
for f in bench_mag_dedup bench_mag_cache; do tail -1 gpurun_out/$f.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$f', d['value'], d['ms_per_step'], d['sampled_edges_per_s'], d['e2e']['value'], d['gpu_launches_per_step'], d['config']['dedup'], d['clocks'])" || tail -5 gpurun_out/$f.log; done
