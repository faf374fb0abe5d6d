# layer-0 owners for dilated nests (C4): parity + A/B
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dilat or C4 or narrow or stress or hostio" > gpurun_out/pytest125.txt 2>&1
for i in 1 2; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C3 | sed "s/^/$v /" >> gpurun_out/ab125.txt 2>&1
done; done
FT_OWNER_L0=0 QT_REPS=50 timeout 300 python tools/quick_time.py C4 | sed "s/^/new_off /" >> gpurun_out/ab125.txt 2>&1
