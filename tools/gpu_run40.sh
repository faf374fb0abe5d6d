for f in 0 1 0 1 0 1; do echo "fast=$f" >> gpurun_out/qt40.log; FT_FAST_GATES=$f QT_REPS=100 QT_WARM=10 timeout 300 python tools/quick_time.py C3 >> gpurun_out/qt40.log 2>&1; done
FT_FAST_GATES=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "bf16" 2>&1 | tail -3 >> gpurun_out/qt40.log
