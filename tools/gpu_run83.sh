# same-box A/B: persisting window off (FT_L2_PERSIST_LAYERS=0) vs default
for i in 1 2 3; do for v in 0 auto; do
  if [ $v = 0 ]; then FT_AB=off FT_L2_PERSIST_LAYERS=0 timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab83.jsonl 2>>gpurun_out/ab83.err;
  else FT_AB=auto timeout 120 python tools/power_probe.py C3 4 >> gpurun_out/ab83.jsonl 2>>gpurun_out/ab83.err; fi
done; done
