# same-box A/B of the default path: libft.so before vs after the tile-counter commit (bench.py)
L=paper_conf_sosp_liuqc0hs0y24_b200/libft.so
for i in 1 2; do for v in old new; do
cp build/ab/libft_$v.so $L
timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['ms_per_step'],3), round(d['value']), d['clocks']['sm_mhz'], d['clocks'].get('power_w_median'))" >> gpurun_out/ab143.txt 2>&1
done; done
cp build/ab/libft_new.so $L
cat gpurun_out/ab143.txt
