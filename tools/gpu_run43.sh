timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "edges or at_least or one_axis or reuse" 2>&1 | tail -15 > gpurun_out/t43.log
