# ncu full capture of the fused tail (one C3 execution) + its source-level stall counters.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"${KREGEX:-k_tail}" -s ${SKIP:-2} -c 1 -o gpurun_out/prof_tail python scripts/run_c3.py C3 4 > gpurun_out/ncu_tail.log 2>&1; echo ncu rc=$?
tail -3 gpurun_out/ncu_tail.log
VARIANTS=default bash scripts/gpu_trace.sh > gpurun_out/trace_all.txt 2>&1; cat gpurun_out/trace_1.txt
