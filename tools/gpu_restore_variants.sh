# sustained relocate (events) of restore build variants: bash tools/gpu_restore_variants.sh "DEF=1" "DEF=2" ...
mkdir -p gpurun_out
TAG=${TAG:-rv}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for V in "$@"; do
  N=$(echo "$V" | tr ' =' '__')
  python - "$V" "$N" <<'PY' || exit 1
import sys
import __graft_entry__ as g
g.build_medusa(out=f"tools/libmedusa_var_{sys.argv[2]}.so", defines=tuple(sys.argv[1].split()))
PY
  MEDUSA_LIB=tools/libmedusa_var_$N.so timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-c5 --no-buffers --sustained 32 > gpurun_out/rv_${TAG}_$N.json 2> gpurun_out/rv_${TAG}_$N.err
  python - gpurun_out/rv_${TAG}_$N.json "$V" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
s = d.get("sustained_relocate", {}); r = d.get("relocate", {}); ip = d.get("relocate_in_place", {})
print(sys.argv[2], "step %.4f ms" % d["ms_per_step"], "sustained x32 %.3f" % s.get("frac_of_peak", 0),
      "in-step %.3f" % r.get("frac_of_peak", 0), "in-place x32 %.3f" % ip.get("x32", {}).get("frac_of_peak", 0))
PY
done
