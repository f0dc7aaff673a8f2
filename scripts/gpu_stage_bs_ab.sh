# A/B: phase-1 CTA size (CUSFFT_STAGE_BS) at equal gathers in flight per SM, C3 bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
for cfg in "256 4 4" "128 4 4" "128 8 2" "128 2 8"; do
set -- $cfg
CUSFFT_STAGE_BS=$1 CUSFFT_STAGE_U=$2 CUSFFT_STAGE_CPS=$3 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_bs$1_u$2_c$3_$rep.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bench_bs$1_u$2_c$3_$rep.json')); print('bs=$1 u=$2 cps(256-thread units)=$3', round(d['value']*1e3,2), 'us gather', round(d['roofline']['kernel_ms']*1e3,2), 'fold', round(d['stage_ms']['fold']*1e3,2), d['accuracy']['exact_recovery'])"
done
done
