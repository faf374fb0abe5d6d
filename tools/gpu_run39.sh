for r in 0 3 5 7 0; do echo "resident=$r" >> gpurun_out/qt39.log; FT_L2_RESIDENT_LAYERS=$r QT_REPS=100 QT_WARM=10 timeout 300 python tools/quick_time.py C3 >> gpurun_out/qt39.log 2>&1; done
