timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio or layer0" > gpurun_out/pytest134.txt 2>&1
