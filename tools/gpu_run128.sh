timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest128.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke128.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench128.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches128.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch128.log 2>&1
