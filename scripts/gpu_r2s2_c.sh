mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_all.log
timeout 300 python scripts/kernel_trace.py gpurun_out/kt_mode2.json --plan-kw "{\"shard_mode\": 2, \"max_hits\": 8192}" > /dev/null 2>gpurun_out/kt.err; echo kt rc=$?
timeout 600 python scripts/scale_model.py gpurun_out/scale_model.json > gpurun_out/scale_model.log 2>&1; echo scale rc=$?
