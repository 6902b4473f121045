"""Per-source-line totals of an ncu source page exported with
--print-source cuda,sass --csv: warp-instructions executed and stall samples,
summed over the SASS of each CUDA line (diagnostic)."""
import csv
import sys

path, top = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30
rows = list(csv.reader(open(path)))
out = {}
src = {}
cur_file = None
hdr = None
last_line = ""
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = {k: i for i, k in enumerate(r)}
        continue
    if hdr is None or len(r) < len(hdr):
        continue
    line = r[0] or last_line
    last_line = line
    if not line:
        continue
    try:
        ie = float(r[hdr["Instructions Executed"]] or 0)
        ss = float(r[hdr["Warp Stall Sampling (All Samples)"]] or 0)
    except ValueError:
        continue
    key = (cur_file, int(line), (r[1] or src.get((cur_file, line), ""))[:90])
    if r[1]:
        src[(cur_file, line)] = r[1]
    a = out.setdefault(key, [0.0, 0.0])
    a[0] += ie
    a[1] += ss
ti = sum(v[0] for v in out.values()) or 1
ts = sum(v[1] for v in out.values()) or 1
print(f"total warp instructions {ti:.0f}, stall samples {ts:.0f}")
print("by instructions:")
for k, v in sorted(out.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{100*v[0]/ti:5.1f}% inst {100*v[1]/ts:5.1f}% stall  {k[0]}:{k[1]}  {k[2]}")
print("by stall samples:")
for k, v in sorted(out.items(), key=lambda kv: -kv[1][1])[:top]:
    print(f"{100*v[0]/ti:5.1f}% inst {100*v[1]/ts:5.1f}% stall  {k[0]}:{k[1]}  {k[2]}")
