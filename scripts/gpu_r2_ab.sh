# A/B of an env switch on the C3 bench value: VARS="CUSFFT_P2_SPC=1 CUSFFT_P2_SPC=2 ..." (two alternations)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "C3_bench or paths_agree or shared_taps or separate" > gpurun_out/pytest_q.log 2>&1; tail -2 gpurun_out/pytest_q.log
for rep in 1 2; do
for v in $VARS; do
  env $v timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/ab_${v}_$rep.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/ab_${v}_$rep.json'))
print('$v', round(d['value']*1e3,2), 'cold', round(d['value_cold']*1e3,2), 'stages', {k: round(v*1e3,2) for k,v in d['stage_ms'].items()}, 'gather', round(d['roofline']['kernel_ms']*1e3,2))"
done; done
