timeout 600 python bench.py --no-cpu-baseline --steps 100 > gpurun_out/bench16.json 2>&1
