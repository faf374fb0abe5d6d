# DSMEM cluster kernel: targeted parity first (bounded), then the suite, then C2 A/B
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "cluster or C2_full" > gpurun_out/pytest91a.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest91.txt 2>&1
for i in 1 2 3; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C2 "C2c:64,128,256,16" "C2h:64,64,128,8" > gpurun_out/ab91_${v}_$i.txt 2>&1
done; done
