# Round-2 check: build, smoke, GPU tests, in-graph trace, bench line, CUPTI kernel trace.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo build rc=$?
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; rc=$?; echo smoke rc=$rc; tail -2 gpurun_out/smoke.log; [ $rc = 0 ] || exit 1
if [ -z "$NO_TESTS" ]; then
timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/pytest_gpu.log
fi
VARIANTS=default bash scripts/gpu_trace.sh > gpurun_out/trace_all.txt 2>&1; cat gpurun_out/trace_1.txt
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
timeout 300 python scripts/kernel_trace.py gpurun_out/kernel_trace.json > /dev/null 2> gpurun_out/kernel_trace.err; echo ktrace rc=$?
echo done
