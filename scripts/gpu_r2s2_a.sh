TESTS=tests TEST_TIMEOUT=1500 bash scripts/gpu_ab_libs.sh "default default:CUSFFT_STAGE_STATIC=100 default:CUSFFT_STAGE_STATIC=50 default:CUSFFT_STAGE_STATIC=90"
timeout 600 python bench.py --steps 20 --ablations --no-cpu-baseline --no-default-line > gpurun_out/bench_abl.json 2> gpurun_out/bench_abl.err; echo abl rc=$?
python -c "import json; d=json.load(open('gpurun_out/bench_abl.json')); print(d['value'], json.dumps(d['ablations']))"
