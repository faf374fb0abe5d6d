for i in 1 2; do
QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 > gpurun_out/qt66_def_$i.txt 2>&1
FT_DEBUG=512 QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 > gpurun_out/qt66_rlx_$i.txt 2>&1
done
FT_DEBUG=512 timeout 300 python tools/event_run.py C4 32 > gpurun_out/ev66.txt 2>&1
timeout 120 python tools/c4_chain.py >> gpurun_out/ev66.txt 2>&1
