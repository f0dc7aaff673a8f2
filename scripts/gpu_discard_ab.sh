# A/B: phase 2's L2 discard of consumed staging lines vs keeping them (the
# next execution's phase-1 stores then hit valid lines: no DRAM write-back).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for d in 1 0; do
CUSFFT_DISCARD=$d timeout 600 ncu --cache-control none --replay-mode application --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:"k_stage|k_fold" -s 6 -c 3 --csv python scripts/flush_probe.py wr 4 > gpurun_out/discard_$d.csv 2>&1; echo ncu d=$d rc=$?
grep -E "k_stage|k_fold" gpurun_out/discard_$d.csv | awk -F'","' '{print $5, $(NF-2), $(NF-1), $NF}' | head -12
done
for rep in 1 2; do
for d in 1 0; do
CUSFFT_DISCARD=$d timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_discard_${d}_$rep.json 2> gpurun_out/bench_discard_${d}_$rep.err; echo bench d=$d rc=$?
python -c "
import json; d=json.load(open('gpurun_out/bench_discard_${d}_$rep.json')); print('d=$d', round(d['value']*1e3,2), 'us gather', round(d['roofline']['kernel_ms']*1e3,2), 'frac', round(d['roofline']['frac'],3), {k: round(v*1e3,2) for k,v in d['stage_ms'].items()}, d['accuracy'])"
done
done
