# same-box A/B of a compile-time variant: epilogue TMEM chunk 8 units (FT_EPI_CH=8) vs 16 (bench.py)
for i in 1 2; do for v in base ch8; do
FT_LIB_PATH=build/ab/libft_$v.so timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['ms_per_step'],3), round(d['value']), d['clocks']['sm_mhz'], d['clocks'].get('power_w_median'))" >> gpurun_out/ab145.txt 2>&1
done; done
for v in base ch8; do FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab145.txt; done
cat gpurun_out/ab145.txt
