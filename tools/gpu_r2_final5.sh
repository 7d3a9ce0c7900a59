# final round-2 state: smoke, full GPU suite, every bench line, reference arm, launch list, ncu
O=gpurun_out/final5; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
lscpu > $O/lscpu.txt; nproc >> $O/lscpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 2000 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
( time timeout 900 python bench.py ) > $O/bench_default.log 2>&1
timeout 400 python bench.py --node-proj off --no-cpu-baseline > $O/bench_GDELT_noproj.log 2>&1
timeout 400 python bench.py --precision bf16 --no-cpu-baseline > $O/bench_GDELT_bf16.log 2>&1
timeout 400 python bench.py --dedup on --precompute on --no-cpu-baseline > $O/bench_GDELT_dedup_pre.log 2>&1
for c in WIKI REDDIT LASTFM MAG; do timeout 600 python bench.py --config $c --no-cpu-baseline > $O/bench_${c}_fp32.log 2>&1; done
( time timeout 900 python bench.py --impl reference ) > $O/ref_default.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_gdelt.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/ncu_launch.log 2>&1
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0 timeout 900 ncu --set full --import-source on --clock-control none -k kv_pre_kernel -s 2 -c 1 -o $O/kv_pre_np_gdelt python tools/kv_probe.py fp32 > $O/ncu_kv.log 2>&1
tail -2 $O/smoke.log; tail -3 $O/pytest_gpu.log
for f in $O/bench_*.log $O/ref_default.log; do echo "$f"; grep metric $f | cut -c1-160; done
