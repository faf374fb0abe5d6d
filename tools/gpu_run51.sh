timeout 300 python tools/lw_event_run.py > gpurun_out/lw_events.jsonl 2>&1
