# Fold issue-order probe + staged-fold mode A/B at C3 (no tests).
mkdir -p gpurun_out
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o scripts/probes/band_probe scripts/probes/band_probe.cu
./scripts/probes/band_probe 1e-7 > gpurun_out/band_probe.txt 2>&1
cat gpurun_out/band_probe.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for v in fused_index fused_scatter split_index split_scatter; do
  CUSFFT_STAGE_MODE=$v timeout 300 python bench.py --no-cpu-baseline --steps 30 > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python -c "import json; d=json.loads(open('gpurun_out/ab_$v.json').readline()); print('$v', round(d['value']*1e3,2), {k: round(v*1e3,2) for k,v in d['stage_ms'].items()})"
done
CUSFFT_NO_STAGE=1 timeout 300 python bench.py --no-cpu-baseline --steps 30 > gpurun_out/ab_nostage.json 2>&1
python -c "import json; d=json.loads(open('gpurun_out/ab_nostage.json').readline()); print('nostage', round(d['value']*1e3,2), {k: round(v*1e3,2) for k,v in d['stage_ms'].items()})"
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"direct|band|stage" -c 10 --csv ./scripts/probes/band_probe > gpurun_out/band_probe_ncu.csv 2>&1
