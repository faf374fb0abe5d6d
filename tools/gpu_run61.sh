timeout 900 python -m pytest tests/test_fused_gather_gpu.py tests/test_gpu_parity.py -x -q -m gpu -k "comm or fused or emulating or layerwise" > gpurun_out/t61.txt 2>&1
