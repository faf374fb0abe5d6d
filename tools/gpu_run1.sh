nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/nproc.txt; lscpu | head -20 >> gpurun_out/nproc.txt
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "f32" -x 2>&1 | tail -30 > gpurun_out/t_f32.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "bf16 and not C3 and not C4 and not C5" 2>&1 | tail -60 > gpurun_out/t_bf16.log
