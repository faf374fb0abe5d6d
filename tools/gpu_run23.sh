timeout 1200 python -m pytest tests/ -m gpu -q 2>&1 | tail -5 > gpurun_out/t23.log
python -c "import __graft_entry__ as g; g.smoke()" >> gpurun_out/t23.log 2>&1
