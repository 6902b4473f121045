"""Summarise an ncu source page (SASS) CSV: top instructions by warp-stall samples."""
import csv
import sys

path, top = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25
rows = list(csv.reader(open(path)))
h = rows[1]
idx = {k: i for i, k in enumerate(h)}
data = [r for r in rows[2:] if len(r) == len(h)]
tot = sum(float(r[idx["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
data.sort(key=lambda r: -float(r[idx["Warp Stall Sampling (All Samples)"]] or 0))
print(f"total samples {tot:.0f}")
for r in data[:top]:
    s = float(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
    print(f"{100*s/tot:5.1f}%  {r[idx['Address']]:>6}  {r[idx['Source']][:90]}")
