# A-operand TMA loads with EVICT_LAST (new default) vs EVICT_NORMAL (FT_DEBUG=4096): DRAM bytes + same-box time
for d in 4096 0; do
FT_DEBUG=$d timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,lts__t_bytes.sum --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu87_d$d.csv 2>&1
done
for i in 1 2 3; do for d in 4096 0; do FT_AB=dbg$d FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab87.jsonl 2>>gpurun_out/ab87.err; done; done
for d in 4096 0; do FT_DEBUG=$d QT_REPS=30 timeout 300 python tools/quick_time.py C4 C5 > gpurun_out/ab87_c45_d$d.txt 2>&1; done
