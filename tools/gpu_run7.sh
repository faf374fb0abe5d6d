timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -5 > gpurun_out/t7.log
timeout 300 python tools/trace_run.py C3 C2 C5 > gpurun_out/trace7.log 2>&1
timeout 300 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt7.log 2>&1
