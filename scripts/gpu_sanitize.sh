# sanitizers are closed on this pool (round 2): this script documents how the r02_sanitize logs were made
# compute-sanitizer memcheck / racecheck / synccheck of the default path (direct launches, no graph)
mkdir -p gpurun_out/sanitize
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
export CUSFFT_NO_GRAPH=1
run() {  # tool name args...
  tool=$1; name=$2; shift 2
  timeout ${SAN_TIMEOUT:-900} compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python scripts/sanitize_run.py "$@" > gpurun_out/sanitize/${tool}_${name}.log 2>&1
  echo "$tool $name rc=$?"; tail -2 gpurun_out/sanitize/${tool}_${name}.log
}
for tool in memcheck racecheck synccheck; do
  run $tool n16_k32 65536 32
  run $tool n16_k32_L24 65536 32 0 L=24 loc_loops=20 vote_threshold=11
  run $tool n22_k1000_staged 4194304 1000
  run $tool n16_k32_B256 65536 32 256
  run $tool n20_k1000_B16384 1048576 1000 16384
  run $tool n18_zero_B16384 262144 64 16384 zero=1
done
run memcheck n22_k1000_chain 4194304 1000 0 gather=1
CUSFFT_TAIL=0 run memcheck n22_k1000_tail0 4194304 1000
