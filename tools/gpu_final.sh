# round-end evidence: tests, smoke, bench (fp32, bf16), launch list, ncu full captures, configs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -x -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_fp32.log 2>&1
timeout 600 python bench.py --precision bf16 --no-cpu-baseline > gpurun_out/bench_bf16.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1
for p in fp32 bf16; do
  PROBE_KV=split PROBE_MASKS=0 TGL_KV=split timeout 600 ncu --set full --import-source on --clock-control none -k regex:kv_split -s 2 -c 1 -o gpurun_out/kv_split_$p python tools/kv_probe.py $p > gpurun_out/ncu_kv_$p.log 2>&1
  python tools/ncu_summary.py gpurun_out/kv_split_$p.ncu-rep > gpurun_out/kv_split_${p}_summary.txt 2>&1
done
CONFIGS="WIKI LASTFM GDELT MAG" TMO=600 bash tools/gpu_configs.sh > gpurun_out/configs.log 2>&1
tail -2 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; cat gpurun_out/configs.log | grep rc=
