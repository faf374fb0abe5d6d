timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" -k "resident or C2 or deterministic or graph or stress" > gpurun_out/par67.txt 2>&1
for i in 1 2 3; do
QT_REPS=50 timeout 300 python tools/quick_time.py C2 > gpurun_out/qt67_new_$i.txt 2>&1
(cd build/oldsrc && QT_REPS=50 timeout 300 python tools/quick_time.py C2) > gpurun_out/qt67_old_$i.txt 2>&1
done
