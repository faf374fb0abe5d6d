timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" -k "grid" > gpurun_out/par69.txt 2>&1
timeout 300 python tools/trace_run.py C5 > gpurun_out/tr69_pair.txt 2>&1
FT_PAIR_CELLS=0 timeout 300 python tools/trace_run.py C5 > gpurun_out/tr69_single.txt 2>&1
