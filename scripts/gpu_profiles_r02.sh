# profiles for round 2: ncu launch list of the bench command, ncu --set full of one C3 execution, plan facts, scale model, CUPTI trace
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
python - > gpurun_out/plan_info.json <<'PY'
import json, sys; sys.path.insert(0, ".")
import bench
from paper_conf_ipps_wangcc16_b200 import Plan, default_B
n, k, L = bench.CONFIGS["C3"][:3]; B = default_B(n, k)
p = Plan(n, k, B=B, L=L, seed=3, **bench.plan_params("C3", B)); i = p.info()
print(json.dumps({"n": n, "k": k, "B": B, "L": L, "w": int(i["w"]), "sum_w": int(i["w"]) * L, "sectors": int(i["sectors"]), **bench.plan_params("C3", B)}))
PY
cat gpurun_out/plan_info.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu-launches rc=$?
timeout 1500 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on -k regex:"k_stage|k_fold|k_fft|k_select|k_tail|k_output" -s 14 -c 7 -o gpurun_out/prof_r02 python scripts/run_c3.py C3 4 > gpurun_out/ncu_all.log 2>&1; echo ncu-full rc=$?
timeout 600 python scripts/scale_model.py gpurun_out/scale_model.json > gpurun_out/scale_model.log 2>&1; echo scale rc=$?; tail -30 gpurun_out/scale_model.log
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace.json --chrome gpurun_out/kernel_trace_chrome.json > /dev/null 2> gpurun_out/kernel_trace.err; echo ktrace rc=$?
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace_cold.json --cold > /dev/null 2>> gpurun_out/kernel_trace.err; echo ktrace-cold rc=$?
