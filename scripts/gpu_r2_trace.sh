mkdir -p gpurun_out
bash scripts/gpu_trace.sh > gpurun_out/trace_all.txt 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
