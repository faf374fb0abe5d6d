# single c-state register array (no spills) + 16-warp epilogue retry: parity + A/B
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest118.txt 2>&1
FT_LIB_PATH=build/ab/libft_e16.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "layer_bands or C3_sampled or small_and_ragged or linear" > gpurun_out/pytest118_e16.txt 2>&1
for i in 1 2; do for v in head new e16; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab118.txt 2>&1
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab118.txt 2>&1
done; done
