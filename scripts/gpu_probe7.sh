# L2 fetch-granularity limit vs random / sorted gathers (C3 shape).
mkdir -p gpurun_out
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o scripts/probes/band_probe scripts/probes/band_probe.cu
./scripts/probes/band_probe 1e-7 > gpurun_out/band_probe2.txt 2>&1
cat gpurun_out/band_probe2.txt
ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:"stage|direct" --csv ./scripts/probes/band_probe 1e-7 > gpurun_out/band_probe2_ncu.csv 2>&1
python3 - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/band_probe2_ncu.csv')) if len(r)>10 and r[0].isdigit()]
for r in rows: print(r[0], r[4][:40], r[-3], r[-1])
PY
