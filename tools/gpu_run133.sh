# split-phase slab pairs (FT_SPLIT_PHASE=1): parity first (bounded), then C3 timing
FT_SPLIT_PHASE=1 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "layer_bands" > gpurun_out/pytest133.txt 2>&1
FT_SPLIT_PHASE=1 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "C3_sampled or hostio" >> gpurun_out/pytest133.txt 2>&1
for i in 1 2; do
SW_REPS=150 timeout 300 python tools/band_sweep.py C3 base FT_SPLIT_PHASE=1 >> gpurun_out/ab133.txt 2>&1
done
timeout 300 python tools/band_sweep.py C3 FT_SPLIT_PHASE=1,FT_BAND=4 FT_TILE_UNITS=32,FT_BAND=4 >> gpurun_out/ab133.txt 2>&1
