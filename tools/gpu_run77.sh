# does the L2 EVICT_LAST weight residency actually cut DRAM reads? (ncu, fixed clock-control none)
for r in 0 4 6; do
FT_L2_RESIDENT_LAYERS=$r timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu77_r$r.csv 2>&1
done
