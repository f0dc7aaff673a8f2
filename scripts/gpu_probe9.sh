mkdir -p gpurun_out
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o scripts/probes/band_probe scripts/probes/band_probe.cu
./scripts/probes/band_probe 1e-7 > gpurun_out/band_probe4.txt 2>&1; cat gpurun_out/band_probe4.txt
