timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "resident" 2>&1 | tail -5 > gpurun_out/t20.log
