# role trace + per-tile event timeline of C3 / C4 after the coalesced-store change
timeout 300 python tools/trace_run.py C3 C4 C2 > gpurun_out/tr79.txt 2>&1
timeout 300 python tools/event_run.py C3 > gpurun_out/ev79.txt 2>&1
timeout 300 python tools/event_analyze.py gpurun_out/events_c3.npy > gpurun_out/eva79.txt 2>&1
