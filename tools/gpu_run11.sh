for d in 3 35 43 51; do echo "FT_DEBUG=$d" >> gpurun_out/qt11.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/qt11.log 2>&1; done
for d in 0 3; do echo "STAGES=7 FT_DEBUG=$d" >> gpurun_out/qt11.log; FT_TRACE_LIB=build/trace/libft_trace7.so FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/qt11.log 2>&1; done
