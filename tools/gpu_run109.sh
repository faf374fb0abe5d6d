# relaxed-scope tempty arrive + per-warp counter release (no CTA barrier before the release): parity + A/B
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest109.txt 2>&1
for i in 1 2; do for v in head new; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab109.txt 2>&1
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 | sed "s/^/$v /" >> gpurun_out/ab109.txt 2>&1
done; done
FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 > gpurun_out/trace109.txt 2>&1
