# A/B of alternative in-tree builds / env settings:
#   bash scripts/gpu_ab_libs.sh "u2 u4:CUSFFT_STAGE_CPS=2 ..." [bench args]
# each spec is lib[:VAR=val[,VAR=val]] (lib -> paper_conf_ipps_wangcc16_b200/libcusfft_<lib>.so)
mkdir -p gpurun_out
SPECS="$1"; shift
if [ -z "$NO_TESTS" ]; then timeout ${TEST_TIMEOUT:-600} python -m pytest ${TESTS:-tests/test_gpu_parity.py} -m gpu -q -x -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_ab.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_ab.log; fi
for rep in 1 2; do for spec in $SPECS; do
  l=${spec%%:*}; envs=""; [ "$spec" != "$l" ] && envs=$(echo ${spec#*:} | tr ',' ' ')
  tag=$(echo "$spec" | tr ':,=' '___')
  lib=libcusfft_$l.so; [ "$l" = default ] && lib=libcusfft.so
  env CUSFFT_LIB=$lib $envs timeout 300 python bench.py --steps 30 --no-cpu-baseline --no-default-line "$@" > gpurun_out/ab_$tag.json 2> gpurun_out/ab_$tag.err
  python - "$tag" <<'PY'
import json, sys
d = json.load(open(f"gpurun_out/ab_{sys.argv[1]}.json"))
r = d["roofline"]; c = d.get("kernels_cupti_us", {})
print(sys.argv[1], "value %.2f us cold %.2f" % (1e3 * d["value"], 1e3 * d["value_cold"]),
      "gather ev %.2f cupti %.2f cold %.2f frac %.3f" % (1e3 * r["kernel_ms"], 1e3 * r["kernel_ms_cupti"], 1e3 * r["kernel_ms_cold"], r["frac"]),
      {k: round(v["mean_us"], 2) for k, v in c.items()}, d["accuracy"]["exact_recovery"])
PY
done; done
