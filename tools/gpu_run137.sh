timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest137.txt 2>&1
QT_REPS=50 timeout 300 python tools/quick_time.py C4 C3 C5 C2 > gpurun_out/qt137.txt 2>&1
