# GDELT tail K|V: ncu --set full of kv_split + ring-depth variants (compile-time)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
CFG=GDELT PROBE_KV=split PROBE_MASKS=0 timeout 600 ncu --set full --import-source on --clock-control none -k regex:kv_split -s 1 -c 1 -o gpurun_out/r02_kv_split_gdelt python tools/kv_probe.py fp32 > gpurun_out/ncu_kv_gdelt.log 2>&1
tail -3 gpurun_out/ncu_kv_gdelt.log
for v in "3 4 2" "5 4 2" "7 2 2" "6 3 2" "4 3 3"; do
  set -- $v
  TGL_NVCC_EXTRA="-DTGL_KV_FSTAGES=$1 -DTGL_KV_BSTAGES=$2 -DTGL_KV_SPLIT_WSTAGES=$3" python -m paper_conf_asplos_wangm24_b200.build -f > /dev/null 2>&1 || { echo "build $v failed"; continue; }
  echo "F=$1 B=$2 W=$3"; CFG=GDELT PROBE_KV=split PROBE_MASKS=0 timeout 300 python tools/kv_probe.py fp32 2>&1 | grep -v "^tail" | tail -1
  CFG=GDELT PROBE_KV=split PROBE_MASKS=0 timeout 300 python tools/kv_probe.py bf16 2>&1 | tail -1
done
python -m paper_conf_asplos_wangm24_b200.build -f > /dev/null 2>&1
