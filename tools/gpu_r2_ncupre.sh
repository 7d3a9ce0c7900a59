# ncu --set full of the kv_pre launch on the GDELT tail block (fp32) + launch list of a GDELT step
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0 timeout 900 ncu --set full --import-source on --clock-control none -k regex:kv_pre -s 2 -c 1 -o gpurun_out/r02_kv_pre_gdelt python tools/kv_probe.py fp32 > gpurun_out/ncu_pre.log 2>&1
tail -3 gpurun_out/ncu_pre.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_gdelt.csv python bench.py --config GDELT --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
tail -2 gpurun_out/ncu_launch.log | cut -c1-200
