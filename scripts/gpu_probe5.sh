mkdir -p gpurun_out
./scripts/probes/gather_probe4 > gpurun_out/gather_probe4.txt 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"direct|phase" -c 6 --csv ./scripts/probes/gather_probe4 > gpurun_out/gather_probe4_ncu.csv 2>&1
