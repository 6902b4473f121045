# ncu --set full of one k_classify launch (ALL10 bench step) + serialized timeline
mkdir -p gpurun_out
TAG=${TAG:-p}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python tools/timeline.py --serial --steps 3 > gpurun_out/tls_$TAG.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_classify -s 3 -c 1 -o gpurun_out/cls_$TAG python bench.py --steps 1 --warmup 3 --sustained 0 --no-cpu-baseline --no-c5 --no-buffers > gpurun_out/ncu_cls_$TAG.log 2>&1
tail -3 gpurun_out/ncu_cls_$TAG.log
