timeout 300 python tools/lw_event_run.py 256,100,1024,4 32,100,1024,4 > gpurun_out/lw_events.jsonl 2>&1
FT_DEBUG=8 timeout 300 python tools/lw_event_run.py 256,100,1024,4 32,100,1024,4 >> gpurun_out/lw_events.jsonl 2>&1
