"""Per-source-line profile of one kernel in an .ncu-rep (needs -lineinfo + --import-source):
instructions executed, stall samples and the top stall reasons, for a line range.

    python tools/ncu_lines.py REP.ncu-rep [first_line last_line] [top]
"""
import collections
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    lo = int(sys.argv[2]) if len(sys.argv) > 3 else 0
    hi = int(sys.argv[3]) if len(sys.argv) > 3 else 10 ** 9
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 60
    import os
    kid = os.environ.get("NCU_KERNEL_ID")        # e.g. ":::2" = the 2nd captured launch
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source",
                          "cuda,sass"] + (["--kernel-id", kid] if kid else []),
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[2]
    ci, si = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    reasons = [k for k, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
    inst, samp, src = collections.Counter(), collections.Counter(), {}
    why = collections.defaultdict(collections.Counter)
    cur, fname = None, ""
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if len(r) < len(h) - 2 or r[0] == "Line No":
            continue
        if r[0]:
            cur = (fname, int(r[0]))
            src[cur] = r[1]
        if not r[2] or r[2] == "-":
            continue
        def f(k):
            try:
                return float(r[k] or 0)
            except ValueError:
                return 0.0
        inst[cur] += f(ci)
        samp[cur] += f(si)
        for k in reasons:
            why[cur][h[k][6:]] += f(k)
    ti, ts = sum(inst.values()) or 1, sum(samp.values()) or 1
    print(f"total warp-instructions {ti:.3g}, stall samples {ts:.0f}")
    sel = [l for l in samp if lo <= l[1] <= hi]
    for l in sorted(sel, key=lambda l: -samp[l])[:top]:
        w = ", ".join(f"{k} {100 * v / max(samp[l], 1):.0f}%" for k, v in why[l].most_common(3) if v)
        print(f"{l[0][:10]:10s}:{l[1]:<5d} inst {100 * inst[l] / ti:5.1f}% stall {100 * samp[l] / ts:5.1f}%  "
              f"{src.get(l, '').strip()[:70]:70s} | {w}")


if __name__ == "__main__":
    main()
