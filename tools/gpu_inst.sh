# per-kernel duration / instructions / DRAM bytes of one bench step (ncu, serialized, cold)
mkdir -p gpurun_out
TAG=${TAG:-x}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none --csv --log-file gpurun_out/inst_$TAG.csv python bench.py --steps 1 --warmup 3 --sustained 0 --no-cpu-baseline > /dev/null 2>&1
python tools/inst_table.py gpurun_out/inst_$TAG.csv
