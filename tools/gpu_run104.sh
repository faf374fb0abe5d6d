# banded C3: DRAM bytes per forward vs band size (is a 4-layer band fully L2-resident?)
for b in 1 2 3 4 5; do
FT_BAND=$b timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu104_b$b.csv 2>&1
done
