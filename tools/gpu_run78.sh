# persisting L2 window for W[0..k): DRAM bytes (ncu) and same-box timing at the power cap
FT_L2_PERSIST_VERBOSE=1 FT_L2_PERSIST_LAYERS=6 timeout 120 python tools/quick_time.py C3 > gpurun_out/q78.txt 2>&1
for k in 0 4 6 8; do
FT_L2_PERSIST_LAYERS=$k timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu78_k$k.csv 2>&1
done
for i in 1 2; do for k in 0 6; do FT_AB=persist$k FT_L2_PERSIST_LAYERS=$k timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab78.jsonl 2>>gpurun_out/ab78.err; done; done
