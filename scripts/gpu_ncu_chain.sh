# ncu full captures of the post-gather chain of one C3 execution (+ source counters)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_fold_fft1_tma|k_fft|k_select|k_tail|k_output|k_stage" -s 14 -c 7 -o gpurun_out/prof_chain python scripts/run_c3.py C3 4 > gpurun_out/ncu_chain.log 2>&1; echo ncu rc=$?
tail -3 gpurun_out/ncu_chain.log
