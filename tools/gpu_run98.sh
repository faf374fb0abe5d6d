# auto layer bands: full GPU suite, C3 auto vs off, strong-scaling batches, role trace
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest98.txt 2>&1
SW_REPS=150 timeout 600 python tools/band_sweep.py C3 FT_BAND=0 base FT_SKEW=2 FT_BAND=0 base > gpurun_out/sweep98.txt 2>&1
for b in 128 64 32; do
SW_REPS=150 timeout 600 python tools/band_sweep.py "b$b:$b,100,1024,16" FT_BAND=0 FT_BAND=4 FT_BAND=8,FT_L2_RESIDENT_LAYERS=16 FT_BAND=2 >> gpurun_out/sweep98.txt 2>&1
done
FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 > gpurun_out/trace98.txt 2>&1
FT_BAND=0 FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace98.txt 2>&1
