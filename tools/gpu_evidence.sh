# ncu evidence + sanitizers + timeline for profiles/ (round tag in $TAG)
mkdir -p gpurun_out
TAG=${TAG:-r1}
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_$TAG.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/gpu_$TAG.txt
# launch list of bench steps (cold, serialised): duration, DRAM bytes, instructions
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --sustained 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_table.py gpurun_out/launches_$TAG.csv > gpurun_out/launch_table_$TAG.txt 2>&1
python tools/make_traffic.py gpurun_out/launches_$TAG.csv gpurun_out/ncu_traffic_$TAG.json > /dev/null
# full capture of the dominant materialize kernel and of restore (a warm step)
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_classify|restore_kernel|restore_inplace_kernel|k_buf_copy" -s 4 -c 5 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 4 --sustained 0 --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
# per-CTA timeline of one graph-captured step
timeout 300 python tools/timeline.py --steps 5 > gpurun_out/timeline_$TAG.txt 2>&1
# sanitizers on the GPU parity tests that use small sets
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_buffers.py -m gpu -x -q -k "toy or tiny or edge or capacity or fault or async or real_memory or errors" > gpurun_out/sanitizer_${tool}_$TAG.log 2>&1
  echo "$tool exit=$?" | tee -a gpurun_out/sanitizer_summary_$TAG.txt
  tail -3 gpurun_out/sanitizer_${tool}_$TAG.log | tee -a gpurun_out/sanitizer_summary_$TAG.txt
done
