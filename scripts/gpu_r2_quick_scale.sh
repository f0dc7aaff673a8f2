bash scripts/gpu_r2_quick.sh
timeout 600 python scripts/scale_model.py gpurun_out/scale_model.json > gpurun_out/scale_model.log 2>&1; echo scale rc=$?; python -c "
import json; d=json.load(open('gpurun_out/scale_model.json'))
for g,v in d['ranks'].items(): print(g, {k: (round(x,1) if isinstance(x,float) else x) for k,x in v.items()})"
