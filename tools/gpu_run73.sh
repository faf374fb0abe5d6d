# power attribution II: fixed-coordinate loads (L2-hot, no DRAM), skip-B, skip epilogue, combos; memory power
for d in 0 32 16 2 34 18; do FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 5 >> gpurun_out/power73.jsonl 2>>gpurun_out/power73.err; done
timeout 120 python tools/power_probe.py gemm 5 >> gpurun_out/power73.jsonl 2>>gpurun_out/power73.err
