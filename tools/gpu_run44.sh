timeout 600 python bench.py --steps 100 > gpurun_out/bench44.json 2> gpurun_out/bench44.err
