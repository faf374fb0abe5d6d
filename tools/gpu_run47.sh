timeout 1500 python tools/depth_sweep.py > gpurun_out/depth_sweep.jsonl 2>&1
