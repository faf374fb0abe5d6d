timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -3 > gpurun_out/t33.log
timeout 300 python tools/event_run.py > gpurun_out/ev33.log 2>&1
timeout 300 python tools/trace_run.py C3 C5 > gpurun_out/trace33.log 2>&1
