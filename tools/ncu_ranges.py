"""Share of instructions / stall samples per source-line range of one kernel.
usage: python tools/ncu_ranges.py report.ncu-rep kernel_regex file name:a-b [name:a-b ...]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep, kre, fname = sys.argv[1:4]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--print-source", "cuda,sass", "--csv", "-k", f"regex:{kre}"],
                     capture_output=True, text=True).stdout
agg = defaultdict(lambda: [0.0, 0.0])
hdr, cur = None, "?"
f = lambda s: float(s) if s not in ("", "-") else 0.0
for row in csv.reader(io.StringIO(out)):
    if not row:
        continue
    if row[0] == "File Path":
        cur = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        hdr = {k: i for i, k in enumerate(row)}
        continue
    if hdr is None or len(row) < len(hdr):
        continue
    try:
        ln = int(row[0])
    except ValueError:
        continue
    try:
        ie, ss = f(row[hdr["Instructions Executed"]]), f(row[hdr["Warp Stall Sampling (All Samples)"]])
    except ValueError:
        continue
    agg[(cur, ln)][0] += ie
    agg[(cur, ln)][1] += ss
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[1] for v in agg.values()) or 1
print(f"instructions {ti:.3g}  samples {ts:.0f}")
for spec in sys.argv[4:]:
    name, r = spec.split(":")
    a, b = map(int, r.split("-"))
    s = [v for k, v in agg.items() if k[0] == fname and a <= k[1] <= b]
    print(f"{name:20s} {100*sum(x[0] for x in s)/ti:5.1f}% inst {100*sum(x[1] for x in s)/ts:5.1f}% smp")
o = [v for k, v in agg.items() if k[0] != fname]
print(f"{'other files':20s} {100*sum(x[0] for x in o)/ti:5.1f}% inst {100*sum(x[1] for x in o)/ts:5.1f}% smp")
