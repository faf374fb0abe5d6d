# same-box A/B: dependency spin on relaxed loads + one acquire (FT_POLL_RELAXED) vs acquire per poll
FT_LIB_PATH=build/ab/libft_pollrlx.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "bands or stress or C3_sampled or C4_sampled or dilated_small or hostio" > gpurun_out/pytest147.txt 2>&1
for i in 1 2 3; do for v in base pollrlx; do
FT_LIB_PATH=build/ab/libft_$v.so timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['ms_per_step'],3), round(d['value']), d['clocks']['sm_mhz'], d['clocks'].get('power_w_median'))" >> gpurun_out/ab147.txt 2>&1
done; done
for v in base pollrlx; do FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=30 timeout 300 python tools/quick_time.py C2 C4 C5 | sed "s/^/$v /" >> gpurun_out/ab147.txt; done
tail -1 gpurun_out/pytest147.txt; cat gpurun_out/ab147.txt
