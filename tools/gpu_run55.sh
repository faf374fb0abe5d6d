timeout 600 python bench.py --steps 100 > gpurun_out/bench55.json 2> gpurun_out/bench55.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches55.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch55.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof55_c3 python tools/quick_time.py C3 > gpurun_out/ncu55.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 -o gpurun_out/prof55_c2 python tools/quick_time.py C2 > gpurun_out/ncu55c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof55_c5 python tools/quick_time.py C5 > gpurun_out/ncu55c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof55_c4 python tools/quick_time.py C4 > gpurun_out/ncu55c4.log 2>&1
