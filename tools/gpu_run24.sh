for d in 0 3 11 19 35 43 51; do echo "FT_DEBUG=$d" >> gpurun_out/trace24.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace24.log 2>&1; done
