mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "batch or k_sweep or variants" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
for p in 1 2 3 4; do
  timeout 600 python bench.py --config C5 --pipeline $p --steps 10 > gpurun_out/c5_p$p.json 2> gpurun_out/c5_p$p.err
  python -c "import json; d=json.loads(open('gpurun_out/c5_p$p.json').readline()); print('C5 pipeline $p', round(d['value']*1e3,2), 'us/transform', d['accuracy'], round(d['e2e']['value']*1e3,1))" || tail -3 gpurun_out/c5_p$p.err
done
