# A/B of fold variants at C3: bench stage times + in-graph kernel spans (trace build).
# VARIANTS: space-separated, each a comma-joined env list ("default" = none).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ipps_wangcc16_b200 import _build
_build.build(force=True, out=_build.OUT.replace('libcusfft.so','libcusfft_trace.so'), defines=['CUSFFT_TRACE'])" >> gpurun_out/build.log 2>&1
if [ -n "$PYTEST_K" ]; then
  env $(echo "$TEST_ENV" | tr ',' ' ') timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "$PYTEST_K" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
  tail -3 gpurun_out/pytest_gpu.log
fi
i=0
for v in ${VARIANTS:-default}; do
  i=$((i+1))
  envs=$(echo "$v" | tr ',' ' '); [ "$v" = default ] && envs=""
  env $envs timeout 300 python bench.py --no-cpu-baseline --steps 30 > gpurun_out/ab_$i.json 2> gpurun_out/ab_$i.err
  python -c "import json; d=json.loads(open('gpurun_out/ab_$i.json').readline()); print('$v', round(d['value']*1e3,2), {k: round(v*1e3,2) for k,v in d['stage_ms'].items()}, d['accuracy']['exact_recovery'])" || tail -3 gpurun_out/ab_$i.err
  env $envs CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py 16 1e-7 8 > gpurun_out/trace_$i.txt 2>&1
  grep -A12 "^kernel" gpurun_out/trace_$i.txt
done
