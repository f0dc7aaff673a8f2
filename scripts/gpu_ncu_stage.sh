# ncu --set full of phase 1 (k_stage_packed) in the bench's steady state: application replay,
# no cache control (the script's own L2 flush precedes every execution, as in bench.py), 6th execution
mkdir -p gpurun_out
python scripts/run_c3.py C3 8 > gpurun_out/plain_c3.log 2>&1 && \
timeout 1500 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on \
  -k regex:"k_stage_packed|k_fft2_select|k_tail|k_output|k_fold_fft1_ms" -s 30 -c 6 -o gpurun_out/prof_r02s2 \
  python scripts/run_c3.py C3 8 > gpurun_out/ncu_stage.log 2>&1; echo ncu rc=$?; tail -3 gpurun_out/ncu_stage.log
