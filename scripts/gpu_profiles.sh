# Evidence for profiles/: launch list of the bench command, one application-replay
# full capture of every kernel of one C3 execution, and the bench line itself.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu-launches rc=$?
timeout 1500 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on -k regex:"k_stage|k_fold|k_fft|k_select|k_vote|k_estimate|k_output" -s 7 -c 7 -o gpurun_out/prof_all python scripts/run_c3.py C3 2 > gpurun_out/ncu_all.log 2>&1; echo ncu-full rc=$?
echo done
