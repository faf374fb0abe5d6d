# 16 epilogue warps (4 per TMEM lane quadrant, 16 units each) vs 8: parity + same-box A/B
FT_LIB_PATH=build/ab/libft_e16.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "bf16 and not layerwise and not b2b and not cluster and not resident" > gpurun_out/pytest102_e16.txt 2>&1
for i in 1 2; do for v in cur e16; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab102.txt 2>&1
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab102.txt 2>&1
done; done
