"""Copy a final GPU run's bench lines into profiles/ (pretty JSON) and print the DESIGN
§12 table rows.  python tools/r02_profiles.py gpurun_out/final4"""
import json
import os
import sys

src = sys.argv[1]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pairs = {"bench_default": "r02_bench_gdelt_fp32", "bench_GDELT_noproj": "r02_bench_gdelt_fp32_noproj",
         "bench_GDELT_bf16": "r02_bench_gdelt_bf16",
         "bench_GDELT_dedup_pre": "r02_bench_gdelt_dedup_pre_fp32",
         "bench_WIKI_fp32": "r02_bench_wiki_fp32", "bench_REDDIT_fp32": "r02_bench_reddit_fp32",
         "bench_LASTFM_fp32": "r02_bench_lastfm_fp32", "bench_MAG_fp32": "r02_bench_mag_fp32",
         "ref_default": "r02_bench_reference_gdelt"}
for s, d in pairs.items():
    try:
        line = [l for l in open(os.path.join(src, s + ".log")) if '"metric"' in l][0]
    except (OSError, IndexError):
        print("missing", s)
        continue
    j = json.loads(line)
    json.dump(j, open(os.path.join(root, "profiles", d + ".json"), "w"), indent=1)
    r = j.get("roofline") or {}
    me = (r.get("method_equivalent") or {}).get("frac")
    e = (j.get("e2e") or {}).get("value")
    print(f"| {d} | {j['value']:.3e} | {j['ms_per_step']:.3f} | "
          f"{(r.get('per_launch_ms') or 0) * 1e3:.0f} | {r.get('frac') or 0:.3f}"
          f"{f' (meq {me:.2f})' if me else ''} | {e or 0:.3e} | "
          f"tcsr {j.get('tcsr', {}).get('build_ms')} cpu {(j.get('cpu_baseline') or {}).get('value')}")
