# coalesced c ring ([H/4][B][4]) + 256-bit h stores: parity, then power attribution of the stores
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest75.txt 2>&1
for d in 0 2048 4096 512; do FT_DEBUG=$d timeout 120 python tools/power_probe.py C3 5 >> gpurun_out/power75.jsonl 2>>gpurun_out/power75.err; done
