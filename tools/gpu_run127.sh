for i in 1 2; do for xd in 0 1; do
FT_X_DIRECT=$xd QT_REPS=50 timeout 300 python tools/quick_time.py C3 C4 | sed "s/^/xd$xd /" >> gpurun_out/ab127.txt 2>&1
done; done
FT_X_DIRECT=1 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "bf16 and not layerwise and not b2b and not cluster and not resident and not grid" > gpurun_out/pytest127.txt 2>&1
