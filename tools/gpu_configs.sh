# one bench line per BASELINE config (single GPU): SURVEY.md §8(d) C2, C3, C5 beside the default ALL10
mkdir -p gpurun_out
TAG=${TAG:-r1}
python -c "import __graft_entry__ as g; g.build()" || exit 1
: > gpurun_out/configs_$TAG.jsonl
for w in qwen1.5-4b llama2-7b llama2-13b all10; do
  timeout 600 python bench.py --workload $w --steps ${STEPS:-50} --warmup 5 --cpu-seconds ${CPU_S:-6} >> gpurun_out/configs_$TAG.jsonl 2> gpurun_out/configs_${TAG}_$w.err
  echo "$w rc=$?"; tail -c 300 gpurun_out/configs_${TAG}_$w.err
done
