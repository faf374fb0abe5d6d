timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -15 > gpurun_out/t_all.log
for r in 0 2 4 6; do echo "resident=$r" >> gpurun_out/qt4.log; FT_L2_RESIDENT_LAYERS=$r timeout 300 python tools/quick_time.py C3 >> gpurun_out/qt4.log 2>&1; done
timeout 300 python tools/quick_time.py C2 C4 C5 >> gpurun_out/qt4.log 2>&1
