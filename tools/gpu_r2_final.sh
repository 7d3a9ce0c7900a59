# round-2 evidence: bench lines per config, reference arm, ncu captures, sanitizer
mkdir -p gpurun_out/final
O=gpurun_out/final
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
lscpu > $O/lscpu.txt; nproc >> $O/lscpu.txt; free -g >> $O/lscpu.txt
( time timeout 900 python bench.py ) > $O/bench_default.log 2>&1
for c in WIKI REDDIT LASTFM MAG; do timeout 900 python bench.py --config $c --no-cpu-baseline > $O/bench_${c}_fp32.log 2>&1; done
timeout 600 python bench.py --config GDELT --precision bf16 --no-cpu-baseline > $O/bench_GDELT_bf16.log 2>&1
timeout 600 python bench.py --config REDDIT --precision bf16 --no-cpu-baseline > $O/bench_REDDIT_bf16.log 2>&1
( time timeout 900 python bench.py --impl reference ) > $O/ref_default.log 2>&1
CFG=GDELT PROBE_KV=pre PROBE_MASKS=0 timeout 900 ncu --set full --import-source on --clock-control none -k regex:kv_pre -s 2 -c 1 -o $O/r02_kv_pre_gdelt_full python tools/kv_probe.py fp32 > $O/ncu_kv.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02_launches_gdelt.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/ncu_launch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02_launches_reddit.csv python bench.py --config REDDIT --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/ncu_launch_r.log 2>&1
timeout 600 compute-sanitizer --tool racecheck python tools/sanitize_attn.py > $O/racecheck.log 2>&1
timeout 600 compute-sanitizer --tool synccheck python tools/sanitize_attn.py > $O/synccheck.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python tools/sanitize_attn.py > $O/memcheck.log 2>&1
tail -3 $O/racecheck.log $O/synccheck.log $O/memcheck.log
for f in $O/bench_*.log $O/ref_default.log; do echo "$f"; grep metric $f | cut -c1-160; done
