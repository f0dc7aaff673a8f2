# ncu launch list of the bench command (cold-cache, serialised: compare SHARES) + the plain run first
mkdir -p gpurun_out
python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/plain_bench.json 2> gpurun_out/plain_bench.err && \
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu rc=$?
