# median ncu duration per kernel name of tools/kv_probe.py (REDDIT tail tgl_tblock_attn)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
PROBE_KV=${KV:-split} PROBE_MASKS=0 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/pk.csv python tools/kv_probe.py ${PREC:-fp32} > /dev/null 2>&1
python - <<'PY'
import csv, statistics
from collections import defaultdict
rows = list(csv.reader(open("gpurun_out/pk.csv")))
hdr, d = None, defaultdict(list)
for r in rows:
    if "Kernel Name" in r: hdr = r; continue
    if hdr and len(r) == len(hdr):
        x = dict(zip(hdr, r)); d[x["Kernel Name"].split("(")[0]].append(float(x["Metric Value"]) / 1000)
for k, v in d.items():
    print(f"{k[:40]:40s} n={len(v):3d} median {statistics.median(v):8.1f} us  min {min(v):8.1f}")
PY
