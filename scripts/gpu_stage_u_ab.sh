# A/B: phase-1 gathers in flight per thread (CUSFFT_STAGE_U) x CTAs per SM (CUSFFT_STAGE_CPS), C3 bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
for cfg in "8 4" "4 4" "4 6" "4 8" "2 8" "2 4" "4 3" "2 6" "4 2"; do
set -- $cfg
CUSFFT_STAGE_U=$1 CUSFFT_STAGE_CPS=$2 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_u$1_c$2_$rep.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bench_u$1_c$2_$rep.json')); print('u=$1 cps=$2', round(d['value']*1e3,2), 'us gather', round(d['roofline']['kernel_ms']*1e3,2), 'fold', round(d['stage_ms']['fold']*1e3,2), d['accuracy']['exact_recovery'])"
done
done
