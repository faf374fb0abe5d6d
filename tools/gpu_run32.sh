timeout 300 python tools/event_run.py > gpurun_out/ev32.log 2>&1
