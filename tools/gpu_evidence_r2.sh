# Round-2 evidence for profiles/: launch lists (ALL10, C5) -> ncu_traffic.json,
# ncu --set full of the top kernels, sustained-relocate DRAM bytes, timelines,
# sanitizers (memcheck, racecheck, synccheck, initcheck) incl. the full-size paths.
mkdir -p gpurun_out
TAG=${TAG:-r2}
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_$TAG.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/gpu_$TAG.txt
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
: > gpurun_out/configs_$TAG.jsonl
for W in qwen1.5-4b llama2-7b llama2-13b all10-inband; do
  timeout 600 python bench.py --workload $W --steps 50 --warmup 5 --cpu-seconds 4 --no-buffers --sustained 8 --c5-sustained 0 >> gpurun_out/configs_$TAG.jsonl 2> gpurun_out/configs_${TAG}_$W.err
done
for W in all10 llama2-13b qwen1.5-4b llama2-7b all10-inband; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_$W.csv python bench.py --workload $W --steps 2 --warmup 3 --sustained 0 --no-cpu-baseline --no-c5 --no-buffers > /dev/null 2>&1
  python tools/make_traffic.py gpurun_out/launches_${TAG}_$W.csv gpurun_out/ncu_traffic_$TAG.json $W > /dev/null
  echo "launch list $W: $(wc -l < gpurun_out/launches_${TAG}_$W.csv) lines"
done
# full captures of the top kernels of an ALL10 step
timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:k_classify|k_iresolve|k_emit|k_rank|restore_kernel" -s 10 -c 5 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 4 --sustained 0 --no-cpu-baseline --no-c5 --no-buffers > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
# sustained relocate (x32) and in place: DRAM bytes per call
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:restore --log-file gpurun_out/sustained_${TAG}.csv python tools/sustained_restore.py > gpurun_out/sustained_${TAG}.json 2> gpurun_out/sustained_${TAG}.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:restore --log-file gpurun_out/sustained_c5_${TAG}.csv python tools/sustained_restore.py --workload llama2-13b --replicas 256 > gpurun_out/sustained_c5_${TAG}.json 2> gpurun_out/sustained_c5_${TAG}.err
# timelines
timeout 300 python tools/timeline.py --steps 5 > gpurun_out/timeline_${TAG}_all10.txt 2>&1
timeout 300 python tools/timeline.py --workload llama2-13b --steps 5 > gpurun_out/timeline_${TAG}_c5.txt 2>&1
timeout 300 python tools/timeline.py --serial --steps 3 > gpurun_out/timeline_${TAG}_serial.txt 2>&1
# sanitizers: every GPU test for memcheck; the full-size and special paths for the others
: > gpurun_out/sanitizer_summary_$TAG.txt
timeout 2400 compute-sanitizer --tool memcheck --report-api-errors no --error-exitcode 9 python -m pytest tests -m gpu -x -q > gpurun_out/sanitizer_memcheck_$TAG.log 2>&1
echo "memcheck (all -m gpu tests) exit=$?" >> gpurun_out/sanitizer_summary_$TAG.txt; tail -3 gpurun_out/sanitizer_memcheck_$TAG.log >> gpurun_out/sanitizer_summary_$TAG.txt
for tool in racecheck synccheck; do
  timeout 1800 compute-sanitizer --tool $tool --report-api-errors no --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_table.py tests/test_gpu_buffers.py tests/test_real_capture.py tests/test_gpu_multi.py -m gpu -x -q -k "all10 or in_place or overflow or real or table or malformed or toy or tiny or edge or capacity or fault or async or every_gpu" > gpurun_out/sanitizer_${tool}_$TAG.log 2>&1
  echo "$tool (full-size + special paths) exit=$?" >> gpurun_out/sanitizer_summary_$TAG.txt
  tail -3 gpurun_out/sanitizer_${tool}_$TAG.log >> gpurun_out/sanitizer_summary_$TAG.txt
done
# initcheck tracks every byte: the small sets, one ALL10 full path, in place, the table cases
# (--check-api-memory-access no: restore writes its output with TMA bulk stores, which initcheck does not
#  track, so every host copy of a restored image would be reported; tests/test_gpu_parity.py
#  test_restore_writes_every_word shows with sentinel-filled destinations that every word is written)
timeout 1800 compute-sanitizer --tool initcheck --check-api-memory-access no --report-api-errors no --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_table.py -m gpu -x -q -p no:cacheprovider -k "(full_path_parity and toy) or (in_place_full_path and toy) or fault or edge_cases or capacity or hand or (chain and toy)" > gpurun_out/sanitizer_initcheck_$TAG.log 2>&1
echo "initcheck (small sets: toy full path, in place, faults, edge cases, capacity, tables, tiny traces, the stream chain) exit=$?" >> gpurun_out/sanitizer_summary_$TAG.txt
tail -3 gpurun_out/sanitizer_initcheck_$TAG.log >> gpurun_out/sanitizer_summary_$TAG.txt
cat gpurun_out/sanitizer_summary_$TAG.txt
