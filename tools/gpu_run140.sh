# A/B: tile-granular dependency counters under the owner walk (FT_TILEDEP) vs whole-cell counters
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "owner_tile_counters or layer_bands" > gpurun_out/pytest140.txt 2>&1
for i in 1 2 3; do for td in 0 1; do
FT_TILEDEP=$td QT_REPS=50 timeout 300 python tools/quick_time.py C3 | sed "s/^/td$td /" >> gpurun_out/ab140.txt 2>&1
done; done
tail -3 gpurun_out/pytest140.txt; cat gpurun_out/ab140.txt
