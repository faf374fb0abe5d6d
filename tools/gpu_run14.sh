for d in 3 35 43 51; do echo "FT_DEBUG=$d" >> gpurun_out/trace14.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace14.log 2>&1; done
