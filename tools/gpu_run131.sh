timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio" > gpurun_out/pytest131.txt 2>&1
FT_HOSTIO_CHUNK=4 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio" >> gpurun_out/pytest131.txt 2>&1
for i in 1 2; do for c in 10 5 3; do
FT_HOSTIO_CHUNK=$c timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench131_c${c}_$i.txt 2>&1
done; done
