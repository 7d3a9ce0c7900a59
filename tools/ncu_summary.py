"""Summarise an .ncu-rep: SOL, memory, scheduler, stall reasons, top SASS hot spots."""
import csv
import io
import subprocess
import sys


def ncu_csv(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, *args, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main(rep, top=25):
    rows = ncu_csv(rep, "--page", "details")
    h = rows[0]
    keep = ("GPU Speed Of Light Throughput", "Memory Workload Analysis", "Scheduler Statistics",
            "Warp State Statistics", "Occupancy", "Compute Workload Analysis", "Launch Statistics")
    for r in rows[1:]:
        d = dict(zip(h, r))
        if d.get("Section Name") in keep and d.get("Metric Name"):
            print(f"{d['Section Name'][:26]:26s} | {d['Metric Name'][:48]:48s} | {d['Metric Value']} {d['Metric Unit']}")
    raw = ncu_csv(rep, "--page", "raw")
    hr, vr = raw[0], raw[2] if len(raw) > 2 else raw[1]
    d = dict(zip(hr, vr))
    print("--- raw")
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
              "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
              "sm__inst_executed_pipe_tensor.sum", "gpu__time_duration.sum"):
        for kk in d:
            if kk.startswith(k):
                print(f"{kk}: {d[kk]}")
    st = [(k, float(v.replace(",", ""))) for k, v in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
          and v.replace(",", "").replace(".", "").isdigit()]
    tot = sum(v for _, v in st) or 1
    print("--- stall samples")
    for k, v in sorted(st, key=lambda x: -x[1])[:10]:
        print(f"{100 * v / tot:5.1f}% {k.replace('smsp__pcsamp_warps_issue_stalled_', '')}")
    src = ncu_csv(rep, "--page", "source", "--print-source", "sass")
    key = "Warp Stall Sampling (All Samples)"
    hs = next((r for r in src if key in r), None)   # one header row per kernel in the report
    if hs is None:
        return
    rs = []
    for x in src[src.index(hs) + 1:]:
        if key in x:                                 # the next kernel's header: stop
            break
        rs.append(dict(zip(hs, x)))

    def f(v):
        try:
            return float(v or 0)
        except ValueError:
            return 0.0
    tot = sum(f(x.get(key)) for x in rs) or 1
    print("--- top SASS by stall samples")
    for x in sorted(rs, key=lambda x: -f(x.get(key)))[:top]:
        print(f"{100 * f(x.get(key)) / tot:5.1f}% {x.get('Address', '')[-5:]} "
              f"{x.get('Source', '').strip()[:90]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
