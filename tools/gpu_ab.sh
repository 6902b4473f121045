# A/B of compile-time variants on the timeline (ALL10 and C5, serial and concurrent)
mkdir -p gpurun_out
TAG=${TAG:-ab}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for V in "$@"; do
  N=$(echo "$V" | tr ' =' '__')
  MEDUSA_DEFINES="$V" timeout 300 python tools/timeline.py --steps 5 > gpurun_out/ab_${TAG}_${N}_all10.txt 2>&1
  MEDUSA_DEFINES="$V" timeout 300 python tools/timeline.py --steps 5 --workload llama2-13b > gpurun_out/ab_${TAG}_${N}_c5.txt 2>&1
  MEDUSA_DEFINES="$V" timeout 300 python tools/timeline.py --steps 3 --serial > gpurun_out/ab_${TAG}_${N}_ser.txt 2>&1
done
