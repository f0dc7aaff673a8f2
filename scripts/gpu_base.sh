mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_all.log
timeout 600 python bench.py --steps 20 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?; tail -2 gpurun_out/bench.err
python -c "
import json; d=json.load(open('gpurun_out/bench.json'))
print('value', d['value'], 'cold', d.get('value_cold'), 'x cuFFT', d.get('speedup_vs_dense_cufft'), d.get('accuracy'))
print('stage', d.get('stage_ms')); print('cupti', d.get('kernels_cupti_us')); r=d['roofline']; print('roof', r)"
