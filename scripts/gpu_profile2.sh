mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for kern in ${KERNS:-k_select k_output k_vote k_fft k_estimate}; do
  timeout 600 ncu --set full --warp-sampling-interval 0 --clock-control none --import-source on -k regex:$kern -s 2 -c 1 -o gpurun_out/prof2_$kern python scripts/run_c3.py C3 3 > gpurun_out/ncu2_$kern.log 2>&1
done
