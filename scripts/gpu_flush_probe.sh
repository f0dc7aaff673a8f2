mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in wr rd none; do
timeout 600 ncu --cache-control none --replay-mode application --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:"k_stage|k_fold" -s 6 -c 3 --csv python scripts/flush_probe.py $m 4 > gpurun_out/flush_$m.csv 2>&1; echo $m rc=$?
grep -E "k_stage|k_fold" gpurun_out/flush_$m.csv | awk -F'","' '{print $5, $(NF-2), $(NF-1), $NF}' | head -12
done
