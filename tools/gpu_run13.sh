for d in 0 3; do echo "FT_DEBUG=$d" >> gpurun_out/trace13.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/trace13.log 2>&1; done
