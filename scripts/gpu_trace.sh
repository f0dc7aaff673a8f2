mkdir -p gpurun_out
CUSFFT_LIB=libcusfft_trace.so python scripts/trace_c3.py 16 > gpurun_out/trace.txt 2>&1
CUSFFT_LIB=libcusfft_trace.so python scripts/trace_c3.py 12 > gpurun_out/trace12.txt 2>&1
