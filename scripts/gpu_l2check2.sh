mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for LL in 4 8 12 16; do
ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct -k regex:"k_stage|k_fold_fft1" -s 4 -c 2 --csv python scripts/run_c3.py C3 4 $LL > gpurun_out/l2check_$LL.csv 2>&1
done
