mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CUSFFT_NO_GRAPH=1 timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -x -k "${PYTEST_K}" > gpurun_out/sanitize.log 2>&1; echo rc=$?
