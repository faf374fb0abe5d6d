timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "130-3-128-2" 2>&1 | grep -E "Error|assert|err" | head -20 > gpurun_out/t28.log
