for i in 1 2; do
for dbg in 0 128; do
FT_DEBUG=$dbg QT_REPS=30 timeout 300 python tools/quick_time.py C3 > gpurun_out/qt57_${dbg}_$i.txt 2>&1
done; done
for dbg in 0 128; do
FT_DEBUG=$dbg timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_op_read_hit_rate.pct --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 python tools/quick_time.py C3 > gpurun_out/ncu57_${dbg}.txt 2>&1
done
