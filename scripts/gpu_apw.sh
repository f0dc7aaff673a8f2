mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import ctypes,torch; from cuda.bindings import runtime as rt; print('maxPersistingL2', rt.cudaDeviceGetAttribute(rt.cudaDeviceAttr.cudaDevAttrMaxPersistingL2CacheSize, 0), 'L2', rt.cudaDeviceGetAttribute(rt.cudaDeviceAttr.cudaDevAttrL2CacheSize, 0))" 2>&1 | tail -1
for v in 1 0; do
CUSFFT_APW=$v timeout 600 ncu --cache-control none --replay-mode application --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct -k regex:"k_stage|k_fold" -s 6 -c 3 --csv python scripts/flush_probe.py wr 4 > gpurun_out/apw_$v.csv 2>&1; echo apw=$v rc=$?
grep -E "k_stage|k_fold" gpurun_out/apw_$v.csv | awk -F'","' '{print substr($5,1,20), $(NF-2), $(NF-1), $NF}' | head -12
done
VARIANTS="default CUSFFT_APW=0 default CUSFFT_APW=0" bash scripts/gpu_ab2.sh 2>&1 | grep -v "^k_\|kernel "
