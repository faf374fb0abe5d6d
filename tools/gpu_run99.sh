# split h/c release + f16x2 gate activations: parity + same-box A/B (banded C3, C4, C5)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest99.txt 2>&1
FT_LIB_PATH=build/ab/libft_splitf16.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "C3_sampled or C4_sampled or C5_sampled or small_and_ragged or C2_full or dilated_small or grid_small or signal or diagnostic" > gpurun_out/pytest99_f16.txt 2>&1
for i in 1 2; do for v in base split f16 splitf16; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab99.txt 2>&1
done; done
for v in base split splitf16; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab99.txt 2>&1
done
