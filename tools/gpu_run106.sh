# owner-computes under layer bands (c in registers, fixed slab -> CTA pair): parity, DRAM bytes, A/B, anatomy
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest106.txt 2>&1
for o in 1 0; do
FT_OWNER=$o timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu106_o$o.csv 2>&1
done
SW_REPS=150 timeout 900 python tools/band_sweep.py C3 base FT_OWNER=0 base FT_OWNER=0 FT_BAND=5 FT_BAND=3 > gpurun_out/ab106.txt 2>&1
FT_L2_RESIDENT_LAYERS=16 timeout 300 python tools/band_events.py C3 64 FT_BAND=4 > gpurun_out/bandev106.txt 2>&1
