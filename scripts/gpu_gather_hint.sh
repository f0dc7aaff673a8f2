mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/ghp scripts/probes/gather_hint_probe.cu
timeout 120 /tmp/ghp > gpurun_out/gather_hint.txt 2>&1; echo rc=$?; cat gpurun_out/gather_hint.txt
