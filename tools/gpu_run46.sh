timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "b2b" 2>&1 | tail -15 > gpurun_out/t46.log
timeout 300 python tools/b2b_time.py >> gpurun_out/t46.log 2>&1
