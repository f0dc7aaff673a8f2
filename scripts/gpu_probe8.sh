# Phase-2 (k_fold_fft1) cost with staging warm vs cold, index vs scatter; ncu without cache flush.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in fused_index fused_scatter; do
  echo "== $m"; CUSFFT_STAGE_MODE=$m python scripts/phase2_probe.py 2>&1 | tail -3
done
for m in fused_index fused_scatter; do
CUSFFT_STAGE_MODE=$m timeout 600 ncu --set full --cache-control none --replay-mode application --clock-control none -k regex:"k_fold|k_stage" -s 4 -c 2 -o gpurun_out/prof_p2_$m python scripts/run_c3.py C3 4 > gpurun_out/ncu_p2_$m.log 2>&1; echo ncu $m rc=$?
done
