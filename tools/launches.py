"""Summarise an ncu launch list (gpu__time_duration.sum per launch) per pipeline step.

A step is the launch sequence from one `batch_roots_kernel` to the next; one-off setup
launches (T-CSR build, time-precompute table, weight packing) fall outside every step.
Prints the per-kernel share of the median step (cold-cache, serialised ncu timings).

    python tools/launches.py launches.csv
"""
import csv
import statistics
import sys
from collections import defaultdict


def main(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            data.append((d["Kernel Name"].split("(")[0][:50], float(d["Metric Value"].replace(",", ""))))
    steps, cur = [], None
    for name, v in data:
        if "batch_roots_kernel" in name:
            if cur:
                steps.append(cur)
            cur = []
        if cur is not None and "Fill" not in name:
            cur.append((name, v))
    # a full step ends with the S14 gather (or, with cache(), the root cache_merge); torch
    # kernels (the bench's per-step counters, outside the timed region) are left out
    # (steps that end at the next batch's roots are complete by construction)
    done = lambda st: any("gather_rows" in n or "cache_merge" in n for n, _ in st)
    if cur and done(cur):
        steps.append(cur)
    steps = [[(n, v) for n, v in s if "at::" not in n and "native::" not in n] for s in steps]
    tot = [sum(v for _, v in s) for s in steps]
    med = sorted(range(len(steps)), key=lambda i: tot[i])[len(steps) // 2]
    s = steps[med]
    agg, cnt = defaultdict(float), defaultdict(int)
    for n, v in s:
        agg[n] += v
        cnt[n] += 1
    T = sum(agg.values())
    print(f"launches={len(data)} steps={len(steps)} median step: {len(s)} launches, {T / 1e3:.1f} us "
          f"(ncu: serialised, cold cache)")
    for n, v in sorted(agg.items(), key=lambda x: -x[1]):
        print(f"{v / 1e3:9.1f} us {100 * v / T:5.1f}% x{cnt[n]:<3d} {n}")


if __name__ == "__main__":
    main(sys.argv[1])
