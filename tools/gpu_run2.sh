timeout 300 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "C3 or C4 or C5" 2>&1 | tail -30 > gpurun_out/t_full.log
