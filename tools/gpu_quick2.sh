# build, GPU tests, timelines (ALL10, C5) and a short bench: the round-2 iteration loop
mkdir -p gpurun_out
TAG=${TAG:-q}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/tests_$TAG.log
timeout 300 python tools/timeline.py --steps 5 > gpurun_out/tl_$TAG.txt 2>&1
timeout 300 python tools/timeline.py --workload llama2-13b --steps 5 > gpurun_out/tl13_$TAG.txt 2>&1
if [ -n "$BENCH" ]; then timeout 900 python bench.py --steps 20 --warmup 5 --no-buffers > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; fi
