# GPU round trip: build, smoke, gpu tests, one bench line (+ optional ncu full capture of named kernels)
mkdir -p gpurun_out
TAG=${TAG:-x}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 400 gpurun_out/bench_$TAG.err
python tools/summarize_bench.py gpurun_out/bench_$TAG.json
if [ -n "$NCU_KERNELS" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$NCU_KERNELS" -s ${NCU_SKIP:-0} -c ${NCU_COUNT:-4} -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 3 --sustained 0 --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
  tail -2 gpurun_out/ncu_$TAG.log
fi
if [ -n "$LAUNCHES" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --sustained 0 --no-cpu-baseline > /dev/null 2>&1
  python tools/launch_table.py gpurun_out/launches_$TAG.csv
fi
