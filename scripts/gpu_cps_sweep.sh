# phase-1 CTAs per SM (CUSFFT_STAGE_CPS) at configs of different gather density: bash scripts/gpu_cps_sweep.sh
for cfg in "--config C4" "--config C5k --k 1000" "--config C5k --k 4096 --bcst 2"; do
for rep in 1 2; do for cps in 4 2 1; do CUSFFT_STAGE_CPS=$cps timeout 600 python bench.py $cfg --steps 10 --no-cpu-baseline --no-default-line --no-cupti > gpurun_out/cps.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/cps.json')); print('$cfg', 'cps', $cps, round(1e3*d['value'],1), round(1e3*d['value_cold'],1), round(1e3*d['stage_ms']['fold'],1))"; done; done; done
