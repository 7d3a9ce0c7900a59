# ncu --set full of the GDELT layer-1 sample launch (132k queries)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sample_kernel -s 1 -c 1 -o gpurun_out/r02_sample_gdelt python bench.py --config GDELT --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_samp.log 2>&1
tail -2 gpurun_out/ncu_samp.log | cut -c1-200
