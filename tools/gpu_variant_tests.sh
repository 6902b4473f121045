# parity tests against build variants: VARIANTS="A=1 B=0;C=1" bash tools/gpu_variant_tests.sh
mkdir -p gpurun_out
TAG=${TAG:-v}
python -c "import __graft_entry__ as g; g.build()" || exit 1
IFS=';' read -ra VS <<< "$VARIANTS"
for V in "${VS[@]}"; do
  N=$(echo "$V" | tr ' =' '__')
  python -c "
import __graft_entry__ as g, sys
g.build_medusa(out='tools/libmedusa_var_$N.so', defines=tuple('$V'.split()))" || exit 1
  MEDUSA_LIB=tools/libmedusa_var_$N.so timeout 900 python -m pytest tests -m gpu -x -q -k "not real_capture" > gpurun_out/vtests_${TAG}_$N.log 2>&1
  echo "$V: $(tail -1 gpurun_out/vtests_${TAG}_$N.log)"
done
