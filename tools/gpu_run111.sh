# owner-computes + skew (input half of (d,t+1) overlaps the epilogue of (d,t))
SW_REPS=150 timeout 900 python tools/band_sweep.py C3 base FT_SKEW=2 FT_SKEW=3 base FT_SKEW=2 FT_SKEW=3 > gpurun_out/ab111.txt 2>&1
FT_SKEW=2 timeout 300 python tools/band_events.py C3 64 FT_BAND=4 > gpurun_out/bandev111.txt 2>&1
timeout 300 python tools/band_events.py C3 64 FT_BAND=4 >> gpurun_out/bandev111.txt 2>&1
