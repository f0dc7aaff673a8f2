# Bench lines of the other BASELINE configs on one B200 (C2, C4, C5 batched at pipeline depths 1-3) + C3.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in C3 C2 C4; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/cfg_$c.json 2> gpurun_out/cfg_$c.err; echo $c rc=$?
  python -c "import json; d=json.loads(open('gpurun_out/cfg_$c.json').readline()); print('$c', round(d['value']*1e3,2), 'us', 'cufft', round(d['dense_cufft_ms']*1e3,1), 'frac', round(d['roofline']['frac'],3), d['roofline']['kernel'][:20], d['accuracy'])" || tail -3 gpurun_out/cfg_$c.err
done
for p in 1 2 3; do
  timeout 900 python bench.py --config C5 --pipeline $p --no-cpu-baseline > gpurun_out/cfg_C5_p$p.json 2> gpurun_out/cfg_C5_p$p.err; echo C5 p$p rc=$?
  python -c "import json; d=json.loads(open('gpurun_out/cfg_C5_p$p.json').readline()); print('C5 p$p', round(d['value']*1e3,2), 'us/transform', {k: d[k] for k in ('accuracy',) if k in d})" || tail -3 gpurun_out/cfg_C5_p$p.err
done
