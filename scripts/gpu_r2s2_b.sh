mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_all.log
timeout 600 python bench.py --steps 20 --ablations --no-cpu-baseline --no-default-line > gpurun_out/bench_abl.json 2> gpurun_out/bench_abl.err; echo abl rc=$?
python -c "import json; d=json.load(open('gpurun_out/bench_abl.json')); print(d['value'], json.dumps(d['ablations']))"
