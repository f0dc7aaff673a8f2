mkdir -p gpurun_out
./scripts/probes/gather_probe > gpurun_out/gather_probe.txt 2>&1
ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,lts__t_requests_srcunit_tex_op_read.sum --clock-control none -k regex:gather --csv ./scripts/probes/gather_probe > gpurun_out/gather_probe_ncu.csv 2>&1
