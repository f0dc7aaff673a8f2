# C4 stage-group size sweep (CUSFFT_STAGE_GROUP): bash scripts/gpu_gs_sweep.sh
for rep in 1 2; do for gs in 4 5 6 3; do CUSFFT_STAGE_GROUP=$gs timeout 600 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-default-line --no-cupti > gpurun_out/gs.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/gs.json')); print('gs', $gs, round(1e3*d['value'],1), round(1e3*d['value_cold'],1), round(1e3*d['stage_ms']['fold'],1))"; done; done
