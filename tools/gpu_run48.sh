timeout 600 python tools/strong_scaling.py > gpurun_out/strong.jsonl 2>&1
