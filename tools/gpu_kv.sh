mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention" -p no:cacheprovider > gpurun_out/pytest_attn.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_attn.log
tail -15 gpurun_out/pytest_attn.log
for kv in bin tma; do
  TGL_KV=$kv timeout 300 python bench.py --no-cpu-baseline --steps 30 > gpurun_out/bench_$kv.log 2>&1
  TGL_KV=$kv timeout 300 python bench.py --no-cpu-baseline --steps 30 --precision bf16 > gpurun_out/bench_${kv}_bf16.log 2>&1
done
for f in gpurun_out/bench_*.log; do echo $f; tail -1 $f | cut -c1-400; done
