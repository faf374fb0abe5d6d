# ring depth: 196 KiB (HEAD: 6 stages at C3) vs the 227 KiB maximum (7 stages); parity first
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest86.txt 2>&1
for i in 1 2 3; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 > gpurun_out/ab86_${v}_$i.txt 2>&1
  FT_AB=$v FT_LIB_PATH=build/ab/libft_$v.so timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab86.jsonl 2>>gpurun_out/ab86.err
done; done
