mkdir -p gpurun_out
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_r1a.json 2> gpurun_out/bench_r1a.err
tail -c 3000 gpurun_out/bench_r1a.json
tail -5 gpurun_out/bench_r1a.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r1a.csv python bench.py --steps 2 --warmup 3 --sustained 0 --no-cpu-baseline > /dev/null 2>&1
wc -l gpurun_out/launches_r1a.csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_classify|restore_kernel|k_check|k_allocs" -s 8 -c 4 -o gpurun_out/prof_r1a python bench.py --steps 1 --warmup 3 --sustained 0 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
ls -la gpurun_out
