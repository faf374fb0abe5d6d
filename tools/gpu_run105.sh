# banded C3: L2 policies (weights / state stores / A loads) x band size: DRAM bytes + timing
for cfg in "4 0" "4 6" "4 10" "4 7" "5 6" "6 6" "5 10"; do set -- $cfg
FT_BAND=$1 FT_L2POL=$2 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:wavefront_bf16 -s 2 -c 1 --csv python tools/quick_time.py C3 > gpurun_out/ncu105_b$1_p$2.csv 2>&1
done
SW_REPS=150 timeout 900 python tools/band_sweep.py C3 base FT_L2POL=6 FT_L2POL=10 FT_L2POL=7 FT_BAND=5,FT_L2POL=6 FT_BAND=6,FT_L2POL=6 FT_BAND=5,FT_L2POL=10 base FT_L2POL=6 > gpurun_out/ab105.txt 2>&1
