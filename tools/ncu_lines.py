"""Aggregate ncu SASS metrics per CUDA source line (mixed cuda,sass page).
usage: python tools/ncu_lines.py report.ncu-rep kernel_regex [top]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
by = sys.argv[4] if len(sys.argv) > 4 else "inst"  # or "smp"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--print-source", "cuda,sass", "--csv", "-k", f"regex:{kre}"],
                     capture_output=True, text=True).stdout
agg = defaultdict(lambda: [0.0, 0.0])
text = {}
cur_file = "?"
hdr = None
for row in csv.reader(io.StringIO(out)):
    if not row:
        continue
    if row[0] == "File Path":
        cur_file = row[1].split("/")[-1]
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
    key = (cur_file, ln)
    text[key] = row[1]
    ie = row[hdr["Instructions Executed"]] if "Instructions Executed" in hdr else ""
    ss = row[hdr["Warp Stall Sampling (All Samples)"]] if "Warp Stall Sampling (All Samples)" in hdr else ""
    try:
        agg[key][0] += float(ie or 0)
        agg[key][1] += float(ss or 0)
    except ValueError:
        pass
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[1] for v in agg.values()) or 1
print(f"instructions {ti:.3g}  samples {ts:.0f}")
for key, (i, s) in sorted(agg.items(), key=lambda kv: -kv[1][0 if by == 'inst' else 1])[:top]:
    print(f"{100*i/ti:5.1f}% inst {100*s/ts:5.1f}% smp  {key[0]}:{key[1]:<5d} {text.get(key, '').strip()[:90]}")
