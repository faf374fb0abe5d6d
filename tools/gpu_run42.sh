timeout 300 python tools/event_run.py C4 32 > gpurun_out/ev42.log 2>&1
