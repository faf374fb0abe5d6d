# owner mode: role trace (epilogue breakdown) + bench + launch list + ncu --set full
FT_TRACE_LIB=build/trace/libft_trace.so timeout 300 python tools/trace_run.py C3 > gpurun_out/trace107.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench107.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches107.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch107.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:wavefront_bf16 -s 2 -c 1 -o gpurun_out/prof107_c3 python tools/quick_time.py C3 > gpurun_out/ncu107.log 2>&1
