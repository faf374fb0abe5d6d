# C5 (grid): DRAM bytes and time vs L2 policies (weights | state stores | A loads)
for pol in 0 7 6 10 11 22 23; do
FT_L2POL=$pol timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C5 > gpurun_out/ncu119_p$pol.csv 2>&1
FT_L2POL=$pol QT_REPS=50 timeout 300 python tools/quick_time.py C5 | sed "s/^/pol$pol /" >> gpurun_out/ab119.txt 2>&1
done
