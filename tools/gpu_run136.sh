for i in 1 2; do for u in 32 64; do
FT_TILE_UNITS=$u QT_REPS=50 timeout 300 python tools/quick_time.py C4 | sed "s/^/u$u /" >> gpurun_out/ab136.txt 2>&1
done; done
for u in 32 64; do
FT_TILE_UNITS=$u QT_REPS=50 timeout 300 python tools/quick_time.py "C4s:256,100,512,6" | sed "s/^/u$u stacked /" >> gpurun_out/ab136.txt 2>&1
done
