TAG=s4 bash tools/gpu_evidence.sh > gpurun_out/evidence_s4.log 2>&1
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_s4.json 2> gpurun_out/bench_s4.err
python tools/summarize_bench.py gpurun_out/bench_s4.json
TAG=s4 bash tools/gpu_configs.sh > gpurun_out/configs_s4.log 2>&1
tail -3 gpurun_out/evidence_s4.log; cat gpurun_out/sanitizer_summary_s4.txt
