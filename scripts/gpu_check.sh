set -x; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
CUSFFT_LIB=libcusfft_trace.so python scripts/trace_c3.py 16 > gpurun_out/trace.txt 2>&1
CUSFFT_BRANCH=1 CUSFFT_LIB=libcusfft_trace.so python scripts/trace_c3.py 16 > gpurun_out/trace_branched.txt 2>&1
if [ -n "$NCU" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu1 rc=$?
fi
