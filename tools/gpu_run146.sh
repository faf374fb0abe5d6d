# final binary of round 2c: bench x2, launch list, ncu --set full of C3, smoke
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke146.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench146.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench146b.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches146.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch146.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof146_c3 python tools/quick_time.py C3 > gpurun_out/ncu146.log 2>&1
tail -1 gpurun_out/smoke146.txt; tail -c 300 gpurun_out/bench146.txt; tail -c 300 gpurun_out/bench146b.txt
