# host-IO overlap: y copied in time chunks by a copy stream that waits on kernel-written counters
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio or layer_bands" > gpurun_out/pytest113.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench113.txt 2>&1
FT_HOSTIO_SERIAL=1 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench113_serial.txt 2>&1
