# build K|V kernel variants (compile-time pipeline depths) and time the REDDIT tail call
mkdir -p gpurun_out
run() {
  TGL_NVCC_EXTRA="$1" python paper_conf_asplos_wangm24_b200/build.py -f > gpurun_out/build_v.log 2>&1 || { echo "build failed: $1"; cat gpurun_out/build_v.log; return; }
  echo "== variant: $1"
  for w in ${WINDOWS:-default}; do
    if [ "$w" = default ]; then unset PROBE_WINDOW; else export PROBE_WINDOW=$w; fi
    for p in ${PRECS:-fp32 bf16}; do
      echo -n "window $w $p: "; PROBE_KV=${KV:-split} PROBE_MASKS=${MASKS:-0} timeout 300 python tools/kv_probe.py $p 2>&1 | grep "mask"
    done
  done
  unset PROBE_WINDOW
}
for v in "$@"; do run "$v"; done
python paper_conf_asplos_wangm24_b200/build.py -f > /dev/null 2>&1
