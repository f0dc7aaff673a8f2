mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for g in -1 32 64 128; do
  python scripts/probe_fetch.py $g > gpurun_out/probe_$g.txt 2>&1
  ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:k_fold -s 4 -c 2 --csv python scripts/probe_fetch.py $g > gpurun_out/probe_ncu_$g.csv 2>&1
done
