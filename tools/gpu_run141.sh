# A/B: whole-cell counters vs tile counters with batched polls (FT_TILEDEP=2)
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "owner_tile_counters" > gpurun_out/pytest141.txt 2>&1
for i in 1 2 3; do for td in 0 2; do
FT_TILEDEP=$td QT_REPS=50 timeout 300 python tools/quick_time.py C3 | sed "s/^/td$td /" >> gpurun_out/ab141.txt 2>&1
done; done
tail -3 gpurun_out/pytest141.txt; cat gpurun_out/ab141.txt
