timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "hostio" > gpurun_out/pytest116.txt 2>&1
for i in 1 2; do
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench116_$i.txt 2>&1
done
