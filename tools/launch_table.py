"""Per-kernel device time of the LAST bench step from an ncu launch list (cold, serialised)."""
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
idx = {k: i for i, k in enumerate(h)}
data = [r for r in rows[1:] if r[idx["Metric Name"]] == "gpu__time_duration.sum"]
names = [r[idx["Kernel Name"]].split("(")[0].split("::")[-1].split("<")[0] for r in data]
vals = [float(r[idx["Metric Value"]]) for r in data]
unit = data[0][idx["Metric Unit"]] if data else "ns"
scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3}[unit]
# one step = from the last 'k_nodes_chunks' to the following 'restore_kernel'
starts = [i for i, n in enumerate(names) if n == "k_trace"]
s = starts[-3] if len(starts) >= 3 else starts[0]  # the timed step (before the e2e loop)
e = next(i for i in range(s, len(names)) if names[i] == "restore_kernel")
tot = 0.0
for i in range(s, e + 1):
    tot += vals[i] * scale
    print(f"  {names[i]:22s} {vals[i]*scale:9.2f} us")
print(f"  {'sum':22s} {tot:9.2f} us")
