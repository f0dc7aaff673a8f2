mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace2.so'), defines=['CUSFFT_TRACE', 'CUSFFT_TRACE_TWICE'])" >> gpurun_out/build.log 2>&1
CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py > gpurun_out/trace_1.txt 2>&1; cat gpurun_out/trace_1.txt
CUSFFT_LIB=libcusfft_trace2.so timeout 300 python scripts/trace_c3.py > gpurun_out/trace_2.txt 2>&1; cat gpurun_out/trace_2.txt
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "C3_bench or paths_agree or dense or overflow or shared_taps" > gpurun_out/pytest_q.log 2>&1; tail -3 gpurun_out/pytest_q.log
