for i in 1 2; do
QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3 > gpurun_out/qt63_new_$i.txt 2>&1
FT_DEBUG=256 QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3 > gpurun_out/qt63_upfront_$i.txt 2>&1
FT_LANES0=0 QT_REPS=30 timeout 300 python tools/quick_time.py C4 > gpurun_out/qt63_nosplit_$i.txt 2>&1
(cd build/oldsrc && QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C3) > gpurun_out/qt63_old_$i.txt 2>&1
done
