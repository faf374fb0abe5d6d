timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" > gpurun_out/par62.txt 2>&1
for i in 1 2; do
QT_REPS=30 timeout 300 python tools/quick_time.py C4 C3 C5 > gpurun_out/qt62_def_$i.txt 2>&1
FT_LANES0=0 QT_REPS=30 timeout 300 python tools/quick_time.py C4 > gpurun_out/qt62_l0_$i.txt 2>&1
done
