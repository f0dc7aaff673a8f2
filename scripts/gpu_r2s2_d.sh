mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "C4 or stage_groups or paths_agree or C5_k_sweep or C3" > gpurun_out/pytest_grp.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_grp.log
for a in "--config C4" "--config C4 --gpus 1 --shard loops" "--config C5k --k 4096 --bcst 2"; do
  timeout 900 python bench.py $a --steps 10 --warmup 3 --no-cpu-baseline --no-default-line > gpurun_out/b.json 2> gpurun_out/b.err; echo "$a rc=$?"
  python -c "
import json; d=json.load(open('gpurun_out/b.json')); r=d['roofline']
print(round(1e3*d['value'],1), 'cold', round(1e3*(d.get('value_cold') or 0),1), 'cufft', d.get('dense_cufft_ms'), 'x', d.get('speedup_vs_dense_cufft'), d['accuracy'])
print(d.get('stage_ms')); print(d.get('kernels_cupti_us')); print(r['kernel'], r['kernel_ms'], r['frac'])"
done
