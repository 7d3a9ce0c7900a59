mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_cache.csv python bench.py --steps 6 --warmup 3 --no-cpu-baseline --cache 1048576 > gpurun_out/bench_ncu_cache.log 2>&1
python tools/launches.py gpurun_out/launches_cache.csv > gpurun_out/step_share_cache.txt 2>&1
head -30 gpurun_out/step_share_cache.txt
