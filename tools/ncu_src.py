"""Summarise an ncu source page (SASS) CSV: top instructions by warp-stall samples."""
import csv
import sys

path, top = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25
rows = list(csv.reader(open(path)))
hi = next(i for i, r in enumerate(rows) if "Address" in r and "Source" in r)
h = rows[hi]
idx = {k: i for i, k in enumerate(h)}
key = "Warp Stall Sampling (All Samples)"
data = [r for r in rows[hi + 1:] if len(r) == len(h) and r[idx["Address"]] != "Address"]
val = lambda r: float(r[idx[key]] or 0)
tot = sum(val(r) for r in data)
print(f"total samples {tot:.0f}")
for r in sorted(data, key=lambda r: -val(r))[:top]:
    print(f"{100*val(r)/tot:5.1f}%  {r[idx['Address']][-5:]:>6}  ie={r[idx['Instructions Executed']]:>8}  {r[idx['Source']][:80]}")
