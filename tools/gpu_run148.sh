# final tree: full GPU suite + smoke
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/suite148.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke148.txt 2>&1
tail -2 gpurun_out/suite148.txt; tail -1 gpurun_out/smoke148.txt
