timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "graph" > gpurun_out/pytest123.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof123_c3 python tools/quick_time.py C3 > gpurun_out/ncu123.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches123.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch123.log 2>&1
