for d in 0 1 2 32 3; do echo "FT_DEBUG=$d" >> gpurun_out/qt38.log; FT_DEBUG=$d QT_REPS=100 QT_WARM=10 timeout 300 python tools/quick_time.py C3 >> gpurun_out/qt38.log 2>&1; done
