# resident kernel: bias in SMEM + single cumulative release — parity and same-box A/B on C2
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest89.txt 2>&1
for i in 1 2 3; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C2 "C2b:128,64,256,8" "C2c:64,128,256,16" > gpurun_out/ab89_${v}_$i.txt 2>&1
done; done
