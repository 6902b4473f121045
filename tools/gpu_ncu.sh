# one ncu --set full capture of the named kernels (regex in $NCU_KERNELS), read back here
mkdir -p gpurun_out
TAG=${TAG:-x}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$NCU_KERNELS" -s ${NCU_SKIP:-0} -c ${NCU_COUNT:-4} -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 3 --sustained 0 --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
tail -3 gpurun_out/ncu_$TAG.log
