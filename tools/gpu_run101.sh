# no-division tile decode + split h/c release (bands only): GPU suite + same-box A/B vs HEAD
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest101.txt 2>&1
for i in 1 2; do for v in head cur; do
  FT_LIB_PATH=build/ab/libft_$v.so SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/$v /" >> gpurun_out/ab101.txt 2>&1
  FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=50 timeout 300 python tools/quick_time.py C4 C5 C2 | sed "s/^/$v /" >> gpurun_out/ab101.txt 2>&1
done; done
for d in 1 2; do
  FT_DEBUG=$d SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base | sed "s/^/dbg$d /" >> gpurun_out/ab101.txt 2>&1
done
