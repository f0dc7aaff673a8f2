mkdir -p gpurun_out
./scripts/probes/gather_probe2 > gpurun_out/gather_probe2.txt 2>&1
ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:"rnd|srt" --csv ./scripts/probes/gather_probe2 > gpurun_out/gather_probe2_ncu.csv 2>&1
