# Round check: build, smoke, GPU tests, bench line, ncu launch list of the bench
# command and one application-replay full capture of one C3 execution.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
if [ -z "$NO_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
fi
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -2 gpurun_out/bench.err
if [ -n "$NCU" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu-launches rc=$?
timeout 1500 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on -k regex:"k_stage|k_fold|k_fft|k_select|k_vote|k_estimate|k_output" -s 9 -c 9 -o gpurun_out/prof_all python scripts/run_c3.py C3 2 > gpurun_out/ncu_all.log 2>&1; echo ncu-full rc=$?
fi
echo done
