# persisting L2 window on by default: full GPU suite, same-box A/B on C3, bench
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest82.txt 2>&1
for i in 1 2 3; do for v in head new; do FT_AB=$v FT_LIB_PATH=build/ab/libft_$v.so timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab82.jsonl 2>>gpurun_out/ab82.err; done; done
timeout 600 python bench.py > gpurun_out/bench82.json 2> gpurun_out/bench82.err
