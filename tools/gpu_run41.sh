timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q 2>&1 | tail -5 > gpurun_out/t41.log
QT_REPS=30 QT_WARM=10 timeout 300 python tools/quick_time.py C4 C3 C5 > gpurun_out/qt41.log 2>&1
FT_TILE_UNITS=64 QT_REPS=30 QT_WARM=10 timeout 300 python tools/quick_time.py C4 >> gpurun_out/qt41.log 2>&1
