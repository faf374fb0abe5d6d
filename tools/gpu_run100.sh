# banded C3 (split release only under bands): GPU suite, bench, launch list, ncu --set full + source
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest100.txt 2>&1
QT_REPS=50 timeout 300 python tools/quick_time.py C3 C4 C2 > gpurun_out/qt100.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench100.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches100.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch100.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof100_c3 python tools/quick_time.py C3 > gpurun_out/ncu100.log 2>&1
