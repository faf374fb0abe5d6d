FT_TRACE_LIB=1 timeout 300 python tools/event_run.py C4 32 > gpurun_out/ev65.txt 2>&1
timeout 120 python tools/c4_chain.py >> gpurun_out/ev65.txt 2>&1
