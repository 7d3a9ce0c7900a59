# per-kernel ncu durations of the REDDIT tail K|V kernel for compile variants x masks
mkdir -p gpurun_out
for v in "$@"; do
  TGL_NVCC_EXTRA="$v" python paper_conf_asplos_wangm24_b200/build.py -f > gpurun_out/build_v.log 2>&1 || { echo "build failed: $v"; tail -20 gpurun_out/build_v.log; continue; }
  PROBE_KV=${KV:-split} PROBE_MASKS=${MASKS:-0,79} timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/pl.csv python tools/kv_probe.py ${PREC:-fp32} > /dev/null 2>&1
  python - "$v" <<'PY'
import csv, os, sys
rows = list(csv.reader(open("gpurun_out/pl.csv")))
hdr, kv = None, []
for r in rows:
    if "Kernel Name" in r: hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if "kv_" in d["Kernel Name"]: kv.append(float(d["Metric Value"]) / 1000)
masks = os.environ.get("MASKS", "0,79").split(",")
kv = kv[2:]                      # the pipeline's own forward: tail + head K|V launches
per = 8                          # kv_probe.py times 8 calls per mask
out = []
for i, m in enumerate(masks):
    seg = kv[i * per + 2:(i + 1) * per]
    out.append(f"mask {m}: {sorted(seg)[len(seg)//2] if seg else float('nan'):.1f} us")
print(f"== {sys.argv[1] or 'default'}: " + "  ".join(out))
PY
done
python paper_conf_asplos_wangm24_b200/build.py -f > /dev/null 2>&1
