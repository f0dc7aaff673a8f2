# Evidence for profiles/: launch list of the bench command and one full capture of the fold.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu-launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fold -s 2 -c 1 -o gpurun_out/prof_fold_full python scripts/run_c3.py C3 3 > gpurun_out/ncu_fold_full.log 2>&1; echo ncu-full rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_stage -s 2 -c 1 -o gpurun_out/prof_k_stage python scripts/run_c3.py C3 3 > gpurun_out/ncu_stage_full.log 2>&1; echo ncu-stage rc=$?
for kern in k_fft k_select k_vote k_estimate k_output; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kern -s 2 -c 1 -o gpurun_out/prof_$kern python scripts/run_c3.py C3 3 > gpurun_out/ncu_$kern.log 2>&1
done
echo done
