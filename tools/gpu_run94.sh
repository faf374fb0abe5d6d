# cluster kernel epilogue: fp32 MUFU activations vs tanh.approx.f16x2 — parity + same-box timing + timeline
FT_LIB_PATH=build/ab/libft_f16m.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "cluster or C2_full" > gpurun_out/pytest94.txt 2>&1
timeout 200 python tools/cluster_events.py 24 > gpurun_out/cev94_24.txt 2>&1
for i in 1 2 3; do for v in f32m f16m; do
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C2 "C2h:64,64,128,8" > gpurun_out/ab94_${v}_$i.txt 2>&1
done; done
