"""One line per kernel launch of an ncu report: duration, DRAM bytes, throughput, occupancy."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                      "gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,"
                      "sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,"
                      "launch__grid_size,launch__block_size,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,"
                      "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,lts__t_sector_hit_rate.pct"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
units = rows[1]
idx = {k: i for i, k in enumerate(h)}
for r in rows[2:]:
    g = lambda k: r[idx[k]] if k in idx else "?"
    name = g("Kernel Name").split("(")[0].split("::")[-1]
    dur = float(g("gpu__time_duration.sum"))
    du = units[idx["gpu__time_duration.sum"]]
    dur_us = {"nsecond": dur / 1000, "ns": dur / 1000, "usecond": dur, "us": dur, "msecond": dur * 1000, "ms": dur * 1000}[du]
    mult = lambda k: {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(units[idx[k]], 1)
    rb = float(g("dram__bytes_read.sum")) * mult("dram__bytes_read.sum")
    wb = float(g("dram__bytes_write.sum")) * mult("dram__bytes_write.sum")
    print(f"{name:18s} {dur_us:9.2f} us  dram R {rb/1e6:8.2f} MB W {wb/1e6:8.2f} MB  "
          f"dram% {g('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed'):>6}  warps% {g('sm__warps_active.avg.pct_of_peak_sustained_active'):>6}  "
          f"regs {g('launch__registers_per_thread')} grid {g('launch__grid_size')}x{g('launch__block_size')} "
          f"bankconf {g('l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum')} l2hit {g('lts__t_sector_hit_rate.pct')}")
