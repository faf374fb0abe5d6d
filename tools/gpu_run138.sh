# final capture of the round: ncu --set full of C3 and C4/C5 summaries, launch list, bench, smoke
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke138.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench138.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches138.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch138.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof138_c3 python tools/quick_time.py C3 > gpurun_out/ncu138.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof138_c4 python tools/quick_time.py C4 > gpurun_out/ncu138_c4.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof138_c5 python tools/quick_time.py C5 > gpurun_out/ncu138_c5.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:wavefront -s 2 -c 1 -o gpurun_out/prof138_c2 python tools/quick_time.py C2 > gpurun_out/ncu138_c2.log 2>&1
