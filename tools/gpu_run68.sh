timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" -k "grid" > gpurun_out/par68.txt 2>&1
for i in 1 2; do
QT_REPS=20 timeout 300 python tools/quick_time.py C5 > gpurun_out/qt68_pair_$i.txt 2>&1
FT_PAIR_CELLS=0 QT_REPS=20 timeout 300 python tools/quick_time.py C5 > gpurun_out/qt68_single_$i.txt 2>&1
done
