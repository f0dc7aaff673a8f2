# quick value / value_cold A/B of in-tree builds on one config: bash scripts/gpu_ab_quick.sh "libs" [bench args]
mkdir -p gpurun_out
LIBS="$1"; shift
for rep in 1 2; do for l in $LIBS; do
  lib=libcusfft_$l.so; [ "$l" = default ] && lib=libcusfft.so
  CUSFFT_LIB=$lib timeout 600 python bench.py --steps 10 --no-cpu-baseline --no-default-line --no-cupti "$@" > gpurun_out/q_$l.json 2> gpurun_out/q_$l.err
  python -c "
import json; d=json.load(open('gpurun_out/q_$l.json'))
print('$l', round(1e3*d['value'],2), 'cold', round(1e3*d['value_cold'],2), {k: round(1e3*v,2) for k, v in d['stage_ms'].items()}, d['accuracy']['exact_recovery'])"
done; done
