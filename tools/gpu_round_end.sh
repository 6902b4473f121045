TAG=s5 bash tools/gpu_evidence.sh > gpurun_out/evidence_s5.log 2>&1
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_s5.json 2> gpurun_out/bench_s5.err
python tools/summarize_bench.py gpurun_out/bench_s5.json
TAG=s5 bash tools/gpu_configs.sh > gpurun_out/configs_s5.log 2>&1
tail -3 gpurun_out/evidence_s5.log; cat gpurun_out/sanitizer_summary_s5.txt
