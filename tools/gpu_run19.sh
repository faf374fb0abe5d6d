timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q 2>&1 | tail -25 > gpurun_out/t19.log
QT_REPS=20 timeout 300 python tools/quick_time.py C2 >> gpurun_out/qt19.log 2>&1
FT_RESIDENT=0 QT_REPS=20 timeout 300 python tools/quick_time.py C2 >> gpurun_out/qt19.log 2>&1
