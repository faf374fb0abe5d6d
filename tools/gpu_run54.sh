timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" > gpurun_out/par54.txt 2>&1
timeout 300 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt54.txt 2>&1
timeout 300 python tools/b2b_time.py > gpurun_out/b2b54.txt 2>&1
timeout 600 python tools/layerwise_time.py > gpurun_out/lw54.jsonl 2>&1
timeout 300 python tools/lw_event_run.py 256,100,1024,4 32,100,1024,4 > gpurun_out/lwev54.jsonl 2>&1
