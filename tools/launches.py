"""Summarise an ncu launch list (gpu__time_duration.sum per launch): last `frac` of launches."""
import csv
import sys
from collections import defaultdict


def main(path, nsteps=3):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    tot, cnt = defaultdict(float), defaultdict(int)
    part = data[-len(data) // nsteps:]
    for d in part:
        n = d["Kernel Name"].split("(")[0][:50]
        tot[n] += float(d["Metric Value"].replace(",", ""))
        cnt[n] += 1
    s = sum(tot.values())
    unit = data[0]["Metric Unit"]
    print(f"launches={len(data)} last-step launches={len(part)} total={s:.0f} {unit}")
    for n, v in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"{v:10.0f} {unit} {100 * v / s:5.1f}% x{cnt[n]:<3d} {n}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 3)
