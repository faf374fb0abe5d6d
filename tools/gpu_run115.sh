timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio" > gpurun_out/pytest115.txt 2>&1
for i in 1 2; do
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench115_$i.txt 2>&1
done
FT_HOSTIO_SERIAL=1 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench115_serial.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest115_all.txt 2>&1
