# end-of-round evidence: smoke, full GPU suite, the default bench line, CUPTI traces (warm / cold),
# the in-graph span trace (trace build), the ncu launch list of the bench command
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_all.log
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo bench rc=$?
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace.json --chrome gpurun_out/kernel_trace_chrome.json > /dev/null 2> gpurun_out/kernel_trace.err; echo ktrace rc=$?
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace_cold.json --cold > /dev/null 2>> gpurun_out/kernel_trace.err; echo ktrace-cold rc=$?
CUSFFT_LIB=libcusfft_trace.so timeout 300 python scripts/trace_c3.py > gpurun_out/trace_c3.txt 2>&1; echo trace rc=$?
python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/plain_bench.json 2> gpurun_out/plain_bench.err && \
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu rc=$?
