timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -3 > gpurun_out/t25.log
for d in 0 3; do echo "FT_DEBUG=$d" >> gpurun_out/trace25.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace25.log 2>&1; done
QT_REPS=30 QT_WARM=10 timeout 300 python tools/quick_time.py C3 C4 C5 > gpurun_out/qt25.log 2>&1
