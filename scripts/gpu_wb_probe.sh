# Staging write-back probe: event times, then per-kernel DRAM bytes under ncu.
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -lineinfo -o /tmp/wb_probe scripts/probes/wb_probe.cu
timeout 120 /tmp/wb_probe > gpurun_out/wb_times.txt 2>&1; echo probe rc=$?
cat gpurun_out/wb_times.txt
timeout 600 ncu --cache-control none --replay-mode application --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:"scatter|readS" --csv /tmp/wb_probe > gpurun_out/wb_ncu.csv 2>&1; echo ncu rc=$?
