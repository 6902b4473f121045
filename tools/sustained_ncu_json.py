"""profiles/<tag>_sustained_relocate_ncu.json from the ncu launch lists of
tools/sustained_restore.py (ALL10 x32 and C5 x256): per launch the duration, DRAM
bytes read / written, DRAM GB/s against the measured HBM peak, algorithmic
bytes and GB/s, and DRAM bytes over algorithmic bytes (diagnostic)."""
import csv
import io
import json
import sys


def rows(csv_path):
    txt = open(csv_path).read()
    lines = [ln for ln in txt.splitlines() if ln.startswith('"')]
    out = {}
    for r in csv.DictReader(io.StringIO("\n".join(lines))):
        k = (int(r["ID"]), r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", ""))
        unit = r["Metric Unit"]
        if r["Metric Name"] == "gpu__time_duration.sum":
            v = v / 1000.0 if unit in ("ns", "nsecond") else (v if unit in ("us", "usecond") else v * 1000.0)
        out.setdefault(k, {})[r["Metric Name"]] = v
    return out


def main():
    res = {}
    for csv_path, json_path in zip(sys.argv[1::2], sys.argv[2::2]):
        meta = json.loads(open(json_path).read().strip().splitlines()[-1])
        lst = []
        for n, ((lid, name), m) in enumerate(sorted(rows(csv_path).items())):
            inplace = "inplace" in name
            alg = meta["alg_bytes_in_place" if inplace else "alg_bytes_out_of_place"]
            us = m["gpu__time_duration.sum"]
            rd, wr = m["dram__bytes_read.sum"], m["dram__bytes_write.sum"]
            kern = name.split("::")[-1].split("(")[0]
            lst.append({"kernel": kern, "launch": n, "us": round(us, 1), "dram_read": rd, "dram_write": wr,
                        "dram_GBs": round((rd + wr) / us / 1e3, 1),
                        "dram_frac_of_peak": round((rd + wr) / us / 1e3 / PEAK, 3),
                        "alg_bytes": alg, "alg_GBs": round(alg / us / 1e3, 1),
                        "alg_frac": round(alg / us / 1e3 / PEAK, 3), "dram_over_alg": round((rd + wr) / alg, 3)})
        res[meta["workload"]] = lst
    res["peak_GBs"] = PEAK
    res["note"] = ("ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                   "--clock-control none over tools/sustained_restore.py; peak = MEASURED_PEAKS.json hbm_gbs")
    print(json.dumps(res, indent=1))


PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"]
if __name__ == "__main__":
    main()
