mkdir -p gpurun_out
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_fp32.log 2>&1
timeout 600 python bench.py --precision bf16 --no-cpu-baseline > gpurun_out/bench_bf16.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1
if [ -n "$NCU_FULL" ]; then
  TGL_KV=split timeout 900 ncu --set full --import-source on --clock-control none -k regex:kv_split -s 2 -c 1 -o gpurun_out/kv_split python tools/kv_probe.py fp32 > gpurun_out/ncu_kv.log 2>&1
  python tools/ncu_summary.py gpurun_out/kv_split.ncu-rep > gpurun_out/kv_split_summary.txt 2>&1
fi
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; tail -1 gpurun_out/bench_fp32.log; tail -1 gpurun_out/bench_bf16.log
