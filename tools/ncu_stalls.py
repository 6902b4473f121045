"""Warp-stall sampling breakdown per kernel launch of an ncu --set full report
(smsp__pcsamp_warps_issue_stalled_* from the raw page), with the executed warp
instructions and issue-active share (diagnostic).
usage: python tools/ncu_stalls.py report.ncu-rep"""
import csv
import io
import subprocess
import sys

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[0]
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    name = d.get("Kernel Name", "?").split("(")[0].split("::")[-1]
    st = {}
    for k, v in d.items():
        if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("_not_issued"):
            try:
                st[k[len("smsp__pcsamp_warps_issue_stalled_"):]] = float(v.replace(",", ""))
            except ValueError:
                pass
    tot = sum(st.values()) or 1.0
    top = sorted(st.items(), key=lambda kv: -kv[1])[:8]
    inst = d.get("smsp__inst_executed.sum", "?")
    act = d.get("smsp__issue_active.avg.pct_of_peak_sustained_active", "?")
    print(f"{name}: warp instructions {inst}, issue active {act}%")
    print("   " + " | ".join(f"{k} {100 * v / tot:.1f}%" for k, v in top))
