# grid (C5) in depth bands: parity, DRAM bytes, timing
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "grid" > gpurun_out/pytest129.txt 2>&1
for b in 0 1 2; do
FT_BAND=$b timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C5 > gpurun_out/ncu129_b$b.csv 2>&1
done
for i in 1 2; do for b in 0 1 2; do
FT_BAND=$b QT_REPS=50 timeout 300 python tools/quick_time.py C5 | sed "s/^/band$b /" >> gpurun_out/ab129.txt 2>&1
done; done
