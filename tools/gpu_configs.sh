# bench.py on every BASELINE config (one GPU), reference arm on REDDIT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in ${CONFIGS:-WIKI LASTFM GDELT MAG}; do
  timeout ${TMO:-900} python bench.py --config $c --steps 20 --warmup 5 --cpu-seconds 20 > gpurun_out/bench_$c.log 2>&1
  echo "$c rc=$?"; tail -1 gpurun_out/bench_$c.log | cut -c1-300
done
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_reference.log 2>&1; tail -1 gpurun_out/bench_reference.log | cut -c1-200
