# final bench line + per-config lines + ALL10 launch list / per-workload ncu counters of the current kernels
mkdir -p gpurun_out
TAG=${TAG:-fin}
python -c "import __graft_entry__ as g; g.build(); g.smoke()" || exit 1
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
: > gpurun_out/configs_$TAG.jsonl
for W in qwen1.5-4b llama2-7b llama2-13b all10-inband; do
  timeout 600 python bench.py --workload $W --steps 50 --warmup 5 --cpu-seconds 4 --no-buffers --sustained 8 --c5-sustained 0 >> gpurun_out/configs_$TAG.jsonl 2> gpurun_out/configs_${TAG}_$W.err
done
for W in all10 llama2-13b qwen1.5-4b llama2-7b all10-inband; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_$W.csv python bench.py --workload $W --steps 2 --warmup 3 --sustained 0 --no-cpu-baseline --no-c5 --no-buffers > /dev/null 2>&1
  python tools/make_traffic.py gpurun_out/launches_${TAG}_$W.csv gpurun_out/ncu_traffic_$TAG.json $W > /dev/null
done
timeout 300 python tools/timeline.py --steps 5 > gpurun_out/timeline_${TAG}_all10.txt 2>&1
timeout 300 python tools/timeline.py --workload llama2-13b --steps 5 > gpurun_out/timeline_${TAG}_c5.txt 2>&1
python tools/summarize_bench.py gpurun_out/bench_$TAG.json | head -4
