# tile-granular dependency counters: parity (incl. stress mode), then same-box A/B vs HEAD
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest80.txt 2>&1
for i in 1 2 3; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 C2 > gpurun_out/ab80_${v}_$i.txt 2>&1
done; done
for i in 1 2; do for v in head new; do FT_AB=$v FT_LIB_PATH=build/ab/libft_$v.so timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab80.jsonl 2>>gpurun_out/ab80.err; done; done
