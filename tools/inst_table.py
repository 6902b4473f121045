"""Per-kernel mean duration, instructions and DRAM bytes from an ncu --csv metrics log
(the last occurrence of each kernel = the last step)."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ix = {k: i for i, k in enumerate(h)}
last = defaultdict(dict)
order = []
for r in rows[1:]:
    if r[ix["ID"]] == "ID":
        continue
    name = r[ix["Kernel Name"]].split("(")[0].split("::")[-1].split("<")[0]
    kid = int(r[ix["ID"]])
    m = r[ix["Metric Name"]]
    try:
        v = float(r[ix["Metric Value"]].replace(",", ""))
    except ValueError:
        continue
    unit = r[ix["Metric Unit"]]
    if m == "gpu__time_duration.sum":
        v = v / 1000.0 if unit in ("ns", "nsecond") else (v * 1000 if unit in ("ms", "msecond") else v)
    last[(name, kid)][m] = v
    if (name, kid) not in order:
        order.append((name, kid))
# keep the last launch of each kernel name
final = {}
for name, kid in order:
    final[name] = last[(name, kid)]
print(f"{'kernel':16s} {'us':>8s} {'Minst':>8s} {'DRAM MB':>8s} {'warps%':>7s}")
tot = [0, 0, 0]
for name, m in final.items():
    us = m.get("gpu__time_duration.sum", 0)
    inst = m.get("smsp__inst_executed.sum", 0) / 1e6
    dram = (m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)) / 1e6
    tot[0] += us; tot[1] += inst; tot[2] += dram
    print(f"{name:16s} {us:8.2f} {inst:8.2f} {dram:8.2f} {m.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):7.1f}")
print(f"{'total':16s} {tot[0]:8.2f} {tot[1]:8.2f} {tot[2]:8.2f}")
