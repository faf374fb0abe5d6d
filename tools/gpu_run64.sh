timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" -k "not slow" > gpurun_out/par64.txt 2>&1
for i in 1 2; do
QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3 > gpurun_out/qt64_new_$i.txt 2>&1
FT_DEBUG=256 QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3 > gpurun_out/qt64_upfront_$i.txt 2>&1
(cd build/oldsrc && QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3) > gpurun_out/qt64_old_$i.txt 2>&1
done
