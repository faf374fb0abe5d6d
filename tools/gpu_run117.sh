# final-state profiles: bench, launch list, ncu --set full of C3, DRAM of C4/C5, role trace
timeout 600 python bench.py > gpurun_out/bench117.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches117.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch117.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof117_c3 python tools/quick_time.py C3 > gpurun_out/ncu117.log 2>&1
for c in C4 C5; do
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__cycles_elapsed.avg.per_second --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py $c > gpurun_out/ncu117_$c.csv 2>&1
done
FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 C4 C5 > gpurun_out/trace117.txt 2>&1
