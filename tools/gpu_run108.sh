FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 > gpurun_out/trace108.txt 2>&1
