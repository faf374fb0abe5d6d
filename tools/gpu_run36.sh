timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q 2>&1 | tail -5 > gpurun_out/t36.log
timeout 300 python tools/trace_run.py C3 C5 > gpurun_out/trace36.log 2>&1
QT_REPS=30 QT_WARM=10 timeout 300 python tools/quick_time.py C3 C4 C5 > gpurun_out/qt36.log 2>&1
