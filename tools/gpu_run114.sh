timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio" > gpurun_out/pytest114.txt 2>&1
for i in 1 2; do
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench114_$i.txt 2>&1
FT_HOSTIO_SERIAL=1 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench114_serial_$i.txt 2>&1
done
