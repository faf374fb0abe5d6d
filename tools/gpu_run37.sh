timeout 600 python bench.py --steps 100 > gpurun_out/bench37.json 2> gpurun_out/bench37.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches37.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch37.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof37_c3 python tools/quick_time.py C3 > gpurun_out/ncu37.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 -o gpurun_out/prof37_c2 python tools/quick_time.py C2 > gpurun_out/ncu37c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof37_c5 python tools/quick_time.py C5 > gpurun_out/ncu37c5.log 2>&1
