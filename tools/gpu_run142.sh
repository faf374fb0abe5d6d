# final state of the round: full GPU suite, smoke, bench, launch list, ncu --set full of C3
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/suite142.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke142.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench142.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches142.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch142.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof142_c3 python tools/quick_time.py C3 > gpurun_out/ncu142.log 2>&1
tail -3 gpurun_out/suite142.txt; tail -2 gpurun_out/smoke142.txt; tail -c 400 gpurun_out/bench142.txt
