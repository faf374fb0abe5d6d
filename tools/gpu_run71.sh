# re-entry confirmation: GPU parity suite, smoke, bench
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest71.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke71.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench71.json 2> gpurun_out/bench71.err
nvidia-smi -q -d POWER > gpurun_out/power71.txt 2>&1
