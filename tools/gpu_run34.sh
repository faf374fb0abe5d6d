timeout 300 python tools/trace_run.py C3 > gpurun_out/trace34.log 2>&1
