"""Summarise an ncu --csv launch list: per launch name, time (us) and DRAM bytes."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
h, by = None, collections.OrderedDict()
for r in rows:
    if r and r[0] == "ID":
        h = r
        continue
    if h and len(r) == len(h):
        d = dict(zip(h, r))
        by.setdefault(d["ID"], {"name": d["Kernel Name"]})[d["Metric Name"]] = d["Metric Value"]
L = list(by.values())[skip:]
for d in L:
    f = lambda k: float(d.get(k, "0").replace(",", "") or 0)
    t = f("gpu__time_duration.sum")
    rb, wb = f("dram__bytes_read.sum"), f("dram__bytes_write.sum")
    print(f"{d['name'][:60]:60s} {t / 1e3:9.1f} us  rd {rb / 1e9:7.2f} GB  wr {wb / 1e9:7.2f} GB"
          + (f"  {(rb + wb) / t:6.0f} GB/s" if t else ""))
