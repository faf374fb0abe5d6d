timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest130.txt 2>&1
QT_REPS=50 timeout 300 python tools/quick_time.py C5 C3 C4 C2 > gpurun_out/qt130.txt 2>&1
