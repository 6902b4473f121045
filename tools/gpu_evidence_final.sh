# final evidence of the current kernels: bench line, per-config lines, launch lists / per-workload ncu
# counters, ncu --set full of the top kernels, sustained-relocate ncu, timelines (no sanitizers: the pool
# refuses compute-sanitizer)
mkdir -p gpurun_out
TAG=${TAG:-fin2}
TAG=$TAG bash tools/gpu_final_bench.sh
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_$TAG.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/gpu_$TAG.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:k_classify|k_iresolve|k_emit|k_rank|restore_kernel" -s 10 -c 5 -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 4 --sustained 0 --no-cpu-baseline --no-c5 --no-buffers > gpurun_out/ncu_$TAG.log 2>&1
tail -1 gpurun_out/ncu_$TAG.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:restore --log-file gpurun_out/sustained_${TAG}.csv python tools/sustained_restore.py > gpurun_out/sustained_${TAG}.json 2> gpurun_out/sustained_${TAG}.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:restore --log-file gpurun_out/sustained_c5_${TAG}.csv python tools/sustained_restore.py --workload llama2-13b --replicas 256 > gpurun_out/sustained_c5_${TAG}.json 2> gpurun_out/sustained_c5_${TAG}.err
timeout 300 python tools/timeline.py --serial --steps 3 > gpurun_out/timeline_${TAG}_serial.txt 2>&1
