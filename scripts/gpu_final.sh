# full GPU suite, the default bench line, CUPTI kernel traces (warm / cold), smoke
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/pytest_all.log
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo bench rc=$?
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace.json --chrome gpurun_out/kernel_trace_chrome.json > /dev/null 2> gpurun_out/kernel_trace.err; echo ktrace rc=$?
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace_cold.json --cold > /dev/null 2>> gpurun_out/kernel_trace.err; echo ktrace-cold rc=$?
