# layer bands / skew of the wavefront order: bitwise vs default order, parity under banding, C3 sweep
FT_BAND=5 FT_SKEW=2 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "C3_sampled or streaming_edges or stress_delayed or narrow_tiles or small_and_ragged or dilated_small" > gpurun_out/pytest96.txt 2>&1
SW_REPS=150 timeout 900 python tools/band_sweep.py C3 base \
  FT_BAND=8 FT_BAND=8,FT_SKEW=2 \
  FT_BAND=6,FT_L2_RESIDENT_LAYERS=16 FT_BAND=6,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=5,FT_L2_RESIDENT_LAYERS=16 FT_BAND=5,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=4,FT_L2_RESIDENT_LAYERS=16 FT_BAND=4,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=5,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16,FT_TILE_UNITS=32 FT_BAND=4,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16,FT_TILE_UNITS=32 \
  FT_BAND=6,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=0,FT_L2_PERSIST_LAYERS=0 FT_BAND=5,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=0,FT_L2_PERSIST_LAYERS=0 \
  base > gpurun_out/sweep96.txt 2>&1
