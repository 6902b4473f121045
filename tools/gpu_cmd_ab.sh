# build + GPU tests + timeline A/B of compile-time variants: TAG=x bash tools/gpu_cmd_ab.sh "A=1" "A=0 B=2" ...
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_$TAG.log 2>&1; echo "tests: $(tail -1 gpurun_out/gputests_$TAG.log)"
bash tools/gpu_ab.sh "$@"
for f in gpurun_out/ab_${TAG}_*; do echo "$f: $(head -1 $f)"; done
