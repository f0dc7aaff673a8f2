mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
for v in 1; do
CUSFFT_TAIL=$v CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py > gpurun_out/trace_t$v.txt 2>&1; head -1 gpurun_out/trace_t$v.txt | tr ' ' '\n' | sort -t: -k2 -n | tr '\n' ' '; echo; tail -9 gpurun_out/trace_t$v.txt
done
