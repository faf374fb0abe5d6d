timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "stress or graph" 2>&1 | tail -20 > gpurun_out/t45.log
