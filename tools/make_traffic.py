"""profiles/ncu_traffic.json from an ncu launch list with dram__bytes_{read,write}.sum:
per-launch DRAM bytes of the last launch of each kernel, keyed by bench.py's names,
stored under the workload the launch list ran (bench.py reads only its own).

  python tools/make_traffic.py LAUNCHES.csv OUT.json WORKLOAD   (OUT.json is merged into)"""
import os
import csv
import json
import sys

NAMES = {"k_classify": "mat_classify", "restore_kernel": "restore", "k_trace": "mat_trace", "k_isort": "mat_isort",
         "report_init": "restore_report_init", "k_result": "mat_result",
         "k_prepare": "mat_prepare", "k_rank": "mat_rank", "k_check_mi": "mat_check_mi",
         "k_check_mm": "mat_check_mm", "k_check": "mat_check", "k_iresolve": "mat_iresolve", "k_emit": "mat_emit", "k_zero": "mat_zero",
         "restore_inplace_kernel": "restore_inplace", "k_buf_copy<true>": "buf_save", "k_buf_copy<false>": "buf_restore"}
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ix = {k: i for i, k in enumerate(h)}
per = {}
inst = {}
for r in rows[1:]:
    if r[ix["ID"]] == "ID":
        continue
    name = r[ix["Kernel Name"]].split("(")[0].split("::")[-1]
    if name not in NAMES:
        name = name.split("<")[0]  # restore_kernel<2> etc.
    if name not in NAMES:
        continue
    m = r[ix["Metric Name"]]
    if m not in ("dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum"):
        continue
    v = float(r[ix["Metric Value"]].replace(",", ""))
    u = r[ix["Metric Unit"]]
    if m == "smsp__inst_executed.sum":
        inst[NAMES[name]] = v * {"inst": 1, "Kinst": 1e3, "Minst": 1e6, "Ginst": 1e9}.get(u, 1)
        continue
    v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
    key = (NAMES[name], int(r[ix["ID"]]))
    per.setdefault(key, 0.0)
    per[key] += v
out = {}
for (bench_name, kid), v in sorted(per.items(), key=lambda kv: kv[0][1]):
    out[bench_name] = v  # the last launch wins
out["_inst"] = inst  # warp instructions per launch (smsp__inst_executed.sum), same launches
out["_note"] = ("per-launch dram__bytes_read.sum + dram__bytes_write.sum of the last bench step in the ncu launch "
                f"list {sys.argv[1].split('/')[-1]} (--clock-control none; ncu flushes caches between launches, so "
                "this is cold-cache traffic)")
wl = sys.argv[3] if len(sys.argv) > 3 else "all10"
allw = json.load(open(sys.argv[2])) if os.path.exists(sys.argv[2]) else {}
allw[wl] = out
json.dump(allw, open(sys.argv[2], "w"), indent=1)
print(json.dumps(out, indent=1))
