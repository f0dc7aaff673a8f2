# A/B of fold-stage variants at C3 (CUSFFT_STAGE_MODE) + GPU parity.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
for v in ${MODES:-fused_index fused_scatter split_index split_scatter}; do
  CUSFFT_STAGE_MODE=$v timeout 300 python bench.py --no-cpu-baseline --steps 30 > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python -c "import json; d=json.loads(open('gpurun_out/ab_$v.json').readline()); print('$v', round(d['value']*1e3,2), {k: round(v*1e3,2) for k,v in d['stage_ms'].items()}, d['gpu_launches'])"
done
if [ -n "$NCU_MODE" ]; then
CUSFFT_STAGE_MODE=$NCU_MODE timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$NCU_MODE.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu-launch rc=$?
CUSFFT_STAGE_MODE=$NCU_MODE timeout 900 ncu --set full --cache-control none --replay-mode application --clock-control none --import-source on -k regex:"k_fold|k_stage|k_fft" -s 6 -c 3 -o gpurun_out/prof_fold_app_$NCU_MODE python scripts/run_c3.py C3 4 > gpurun_out/ncu_fold_app.log 2>&1; echo ncu-fold rc=$?
fi
