mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for kern in k_fft k_select k_vote k_estimate k_output k_fold; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kern -s 2 -c 1 -o gpurun_out/prof_$kern python scripts/run_c3.py C3 3 > gpurun_out/ncu_$kern.log 2>&1
done
