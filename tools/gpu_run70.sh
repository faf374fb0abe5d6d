timeout 300 python tools/trace_run.py C5 > gpurun_out/tr70_base.txt 2>&1
FT_DEBUG=1 timeout 300 python tools/trace_run.py C5 > gpurun_out/tr70_nodeps.txt 2>&1
FT_DEBUG=3 timeout 300 python tools/trace_run.py C5 > gpurun_out/tr70_nodeps_noepi.txt 2>&1
FT_DEBUG=33 timeout 300 python tools/trace_run.py C5 > gpurun_out/tr70_nodeps_fixed.txt 2>&1
