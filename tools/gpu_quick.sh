# quick GPU check: build, GPU parity tests, a short bench (no CPU baseline / sustained), summary
mkdir -p gpurun_out
TAG=${TAG:-q}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -4
timeout 600 python bench.py --steps ${STEPS:-30} --warmup 5 --no-cpu-baseline --sustained ${SUST:-0} > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 600 gpurun_out/bench_$TAG.err
python tools/summarize_bench.py gpurun_out/bench_$TAG.json > gpurun_out/sum_$TAG.txt 2>&1; cat gpurun_out/sum_$TAG.txt
