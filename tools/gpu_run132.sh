FT_LIB_PATH=build/ab/libft_f16.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "C3_sampled or C4_sampled or C5_sampled or layer_bands or signal or diagnostic or small_and_ragged" > gpurun_out/pytest132_f16.txt 2>&1
for i in 1 2; do for v in cur f16; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab132.txt 2>&1
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab132.txt 2>&1
done; done
