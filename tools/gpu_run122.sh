timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke122.txt 2>&1
for b in 128 64 32; do
SW_REPS=150 timeout 600 python tools/band_sweep.py "b$b:$b,100,1024,16" base FT_BAND=4 FT_BAND=6 FT_BAND=8 >> gpurun_out/sweep122.txt 2>&1
done
