# power / clock attribution: cuBLAS GEMM vs C3 and C3 with parts switched off (FT_DEBUG bits)
nvidia-smi -q -d PERFORMANCE,POWER,CLOCK,TEMPERATURE > gpurun_out/smi72_before.txt 2>&1
for m in gemm C3; do timeout 120 python tools/power_probe.py $m 6 >> gpurun_out/power72.jsonl 2>>gpurun_out/power72.err; done
for d in 2 16 8 24 1; do FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 6 >> gpurun_out/power72.jsonl 2>>gpurun_out/power72.err; done
timeout 120 python tools/power_probe.py gemm 6 >> gpurun_out/power72.jsonl 2>>gpurun_out/power72.err
nvidia-smi -q -d PERFORMANCE,POWER,CLOCK,TEMPERATURE > gpurun_out/smi72_after.txt 2>&1
