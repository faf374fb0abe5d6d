# round-1 re-entry: full GPU suite, smoke, default bench, C2-C5 quick timings
nvidia-smi --query-gpu=name,clocks.max.sm,power.limit --format=csv > gpurun_out/smi95.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest95.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/smoke95.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench95.txt 2>&1
QT_REPS=30 timeout 600 python tools/quick_time.py C2 C3 C4 C5 > gpurun_out/qt95.txt 2>&1
