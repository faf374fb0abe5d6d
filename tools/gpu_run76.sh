# same-box A/B: HEAD (c ring [B][H], 128-bit h stores) vs new (c ring [H/4][B][4], 256-bit h stores)
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest76.txt 2>&1
for i in 1 2 3; do
  for v in head new; do FT_AB=$v FT_LIB_PATH=build/ab/libft_$v.so timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab76.jsonl 2>>gpurun_out/ab76.err; done
done
