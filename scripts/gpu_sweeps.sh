# BASELINE.json configs on one B200: C1, C2, C4 (SNR sweep), the C5 k sweep and the C5 batch (JSON lines -> gpurun_out/configs/)
mkdir -p gpurun_out/configs
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
B="timeout 600 python bench.py --steps 20 --no-cupti --no-default-line"
$B --config C1 > gpurun_out/configs/C1.json 2> gpurun_out/configs/C1.err; echo C1 $?
$B --config C2 --no-cpu-baseline > gpurun_out/configs/C2.json 2> gpurun_out/configs/C2.err; echo C2 $?
for snr in none 60 40 20 10 0; do
  if [ $snr = none ]; then a=""; else a="--snr $snr"; fi
  $B --config C4 --no-cpu-baseline $a > gpurun_out/configs/C4_snr$snr.json 2> gpurun_out/configs/C4_snr$snr.err; echo C4 $snr $?
done
for k in 50 100 200 500 1000 2000 4096; do
  bc=1.0; [ $k -ge 2000 ] && bc=2.0
  $B --config C5k --k $k --bcst $bc --no-cpu-baseline > gpurun_out/configs/C5k_$k.json 2> gpurun_out/configs/C5k_$k.err; echo C5k $k $?
done
timeout 600 python bench.py --config C5 --steps 10 > gpurun_out/configs/C5_batch.json 2> gpurun_out/configs/C5_batch.err; echo C5 $?
python - <<'PY'
import json, glob, os
for f in sorted(glob.glob("gpurun_out/configs/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(os.path.basename(f), "ERR", e); continue
    acc = d.get("accuracy", {})
    print(f"{os.path.basename(f):18s} {d['value']*1e3:9.1f} us  cuFFT {d.get('dense_cufft_ms', 0)*1e3:8.1f} us  x{d.get('speedup_vs_dense_cufft', 0):5.2f}  exact={acc.get('exact_recovery')} l1={acc.get('l1_per_coefficient')}")
PY
