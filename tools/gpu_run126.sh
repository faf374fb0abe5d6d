timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "layer0_owner or dilat or C4" > gpurun_out/pytest126.txt 2>&1
QT_REPS=50 timeout 300 python tools/quick_time.py C4 C3 C5 C2 > gpurun_out/qt126.txt 2>&1
