# power attribution III: epilogue stores vs gate math; L2-resident layers
for d in 0 512 1024 1536; do FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 5 >> gpurun_out/power74.jsonl 2>>gpurun_out/power74.err; done
for r in 4 7; do FT_L2_RESIDENT_LAYERS=$r timeout 120 python tools/power_probe.py C3 5 >> gpurun_out/power74.jsonl 2>>gpurun_out/power74.err; done
