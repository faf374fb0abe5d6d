# round-2 profiles of the current kernels: ncu --set full (C3, C4, C5, C2) + the bench launch list
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches85.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch85.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof85_c3 python tools/quick_time.py C3 > gpurun_out/ncu85.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof85_c4 python tools/quick_time.py C4 > gpurun_out/ncu85c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof85_c5 python tools/quick_time.py C5 > gpurun_out/ncu85c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 -o gpurun_out/prof85_c2 python tools/quick_time.py C2 > gpurun_out/ncu85c2.log 2>&1
