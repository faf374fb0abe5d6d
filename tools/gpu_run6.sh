timeout 300 python tools/trace_run.py C3 C2 C5 > gpurun_out/trace6.log 2>&1
