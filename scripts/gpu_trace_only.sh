# build the trace library and print the C3 in-graph trace (ARGS: trace_c3.py arguments)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py ${ARGS} > gpurun_out/trace_1.txt 2>&1; cat gpurun_out/trace_1.txt
