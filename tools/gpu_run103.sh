# banded C3: L2 policy of the nest state (hb / c ring stores): EVICT_LAST (default) vs EVICT_NORMAL (FT_DEBUG=128)
SW_REPS=150 timeout 600 python tools/band_sweep.py C3 base FT_DEBUG=128 base FT_DEBUG=128 > gpurun_out/ab103.txt 2>&1
for d in 0 128; do
FT_DEBUG=$d timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu103_d$d.csv 2>&1
done
