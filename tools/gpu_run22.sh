timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "linear" 2>&1 | tail -25 > gpurun_out/t22.log
