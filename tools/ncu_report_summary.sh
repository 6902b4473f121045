# profiles/<tag>_ncu_summary.txt from an ncu --set full report + SASS evidence + box info
# usage: bash tools/ncu_report_summary.sh gpurun_out/prof_X.ncu-rep gpurun_out/gpu_X.txt "header line"
REP=$1; BOX=$2; HDR=$3
echo "# $HDR"
python tools/ncu_summary.py "$REP"
echo
echo "# SASS evidence (cuobjdump -sass paper_conf_asplos_zengxgcl25_b200/libmedusa.so)"
for m in UBLKCP UBLKPF SYNCS.ARRIVE.TRANS64 SYNCS.PHASECHK ACQBULK PREEXIT REDUX ATOMG ATOMS; do
  echo "$m: $(cuobjdump -sass paper_conf_asplos_zengxgcl25_b200/libmedusa.so | grep -c "$m")"
done
echo
echo "# GPU box"
cat "$BOX"
ncu -i "$REP" --page details --csv 2>/dev/null | python3 -c '
import csv, sys
want = {"Memory Throughput", "DRAM Throughput", "Duration", "L2 Cache Throughput", "Executed Ipc Active",
        "Issue Slots Busy", "L2 Hit Rate", "No Eligible", "Registers Per Thread", "Theoretical Occupancy",
        "Achieved Occupancy", "Waves Per SM"}
for r in csv.reader(sys.stdin):
    if len(r) > 14 and r[12] in want:
        print(f"{r[4][:30]} | {r[12]} {r[14]} {r[13]}")
'
