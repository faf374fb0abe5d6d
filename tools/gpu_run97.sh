# banded order: event anatomy (trace build) + more sweep points
for s in "FT_BAND=4 FT_SKEW=1" "FT_BAND=4 FT_SKEW=2" "FT_BAND=6 FT_SKEW=2" "FT_BAND=0 FT_SKEW=1"; do
  FT_L2_RESIDENT_LAYERS=16 timeout 300 python tools/band_events.py C3 64 $s >> gpurun_out/bandev97.txt 2>&1
done
SW_REPS=150 timeout 900 python tools/band_sweep.py C3 base \
  FT_BAND=4,FT_L2_RESIDENT_LAYERS=16 FT_BAND=4,FT_SKEW=3,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=3,FT_L2_RESIDENT_LAYERS=16 FT_BAND=3,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=16,FT_SKEW=2 FT_BAND=7,FT_SKEW=2,FT_L2_RESIDENT_LAYERS=16 \
  FT_BAND=4,FT_L2_RESIDENT_LAYERS=16 base > gpurun_out/sweep97.txt 2>&1
