# In-graph per-kernel spans (trace build).  VARIANTS: space-separated env
# assignments joined by commas, e.g. "CUSFFT_P2_SPC=1 CUSFFT_P2_SPC=2,CUSFFT_FORK=0".
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
i=0
for v in ${VARIANTS:-default}; do
  i=$((i+1))
  envs=$(echo "$v" | tr ',' ' ')
  [ "$v" = default ] && envs=""
  echo "=== variant $v"
  env $envs CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py 16 1e-7 8 > gpurun_out/trace_$i.txt 2>&1
  cat gpurun_out/trace_$i.txt
done
