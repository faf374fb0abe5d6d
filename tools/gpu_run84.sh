# energy attribution: no MMAs (FT_DEBUG=4), no MMAs + no weight loads (20), baseline
for d in 0 4 20; do FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/power84.jsonl 2>>gpurun_out/power84.err; done
