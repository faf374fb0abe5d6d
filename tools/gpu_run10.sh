for d in 3 7 15 23 11 19; do echo "FT_DEBUG=$d" >> gpurun_out/qt10.log; FT_DEBUG=$d timeout 300 python tools/trace_run.py C3 >> gpurun_out/qt10.log 2>&1; done
