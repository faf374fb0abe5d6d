timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "layer_bands" > gpurun_out/pytest110.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench110.txt 2>&1
