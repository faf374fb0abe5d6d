timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -5 > gpurun_out/t15.log
for d in 0 3; do echo "FT_DEBUG=$d" >> gpurun_out/trace15.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace15.log 2>&1; done
timeout 300 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt15.log 2>&1
