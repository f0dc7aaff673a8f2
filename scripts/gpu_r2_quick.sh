# quick loop: build, trace build + C3 trace, focused GPU tests, short bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py > gpurun_out/trace_1.txt 2>&1; head -1 gpurun_out/trace_1.txt | tr ' ' '\n' | sort -t: -k2 -n | tr '\n' ' '; echo; tail -8 gpurun_out/trace_1.txt
timeout ${TEST_TIMEOUT:-600} python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider ${PYTEST_ARGS:--k "C3_bench or paths_agree or dense or overflow or shared_taps or separate or batch"} > gpurun_out/pytest_q.log 2>&1; tail -3 gpurun_out/pytest_q.log
timeout 600 python bench.py --steps 20 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?; tail -2 gpurun_out/bench.err
python -c "
import json; d=json.load(open('gpurun_out/bench.json'))
print('value', d['value'], 'cold', d['value_cold'], 'x cuFFT', d['speedup_vs_dense_cufft'], d['accuracy'])
print('stage', d['stage_ms']); print('cupti', d['kernels_cupti_us']); r=d['roofline']; print('roof', r['kernel_ms'], r['frac'], r['kernel_ms_cold'])"
