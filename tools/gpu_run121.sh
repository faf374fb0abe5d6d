timeout 1500 python tools/depth_sweep.py > gpurun_out/depth_sweep121.jsonl 2>&1
timeout 600 python tools/layerwise_time.py > gpurun_out/lw121.jsonl 2>&1
timeout 600 python tools/strong_scaling.py > gpurun_out/strong121.jsonl 2>&1
