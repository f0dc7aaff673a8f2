# Full GPU tests + bench + ncu (no cache flush, application replay) of the post-fold chain kernels.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
python -c "import json; d=json.loads(open('gpurun_out/bench.json').readline()); print(d['value'], d['stage_ms'], d['roofline']['frac'], d['speedup_vs_dense_cufft'])"
timeout 900 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on -k regex:"k_fft|k_select|k_vote|k_estimate|k_output|k_fold_fft1_tma|k_stage" -s 14 -c 7 -o gpurun_out/prof_chain python scripts/run_c3.py C3 6 > gpurun_out/ncu_chain.log 2>&1; echo ncu rc=$?
