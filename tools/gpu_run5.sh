timeout 300 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt5.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench5.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof5_c3 python tools/quick_time.py C3 > gpurun_out/ncu5.log 2>&1
