mkdir -p gpurun_out
./scripts/probes/gather_probe3 > gpurun_out/gather_probe3.txt 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"phase" --csv ./scripts/probes/gather_probe3 > gpurun_out/gather_probe3_ncu.csv 2>&1
