# re-entry validation of the restored tree: full GPU suite, smoke, bench, reference arm
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/suite139.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke139.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench139.txt 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/ref139.txt 2>&1
tail -3 gpurun_out/suite139.txt; tail -2 gpurun_out/smoke139.txt; tail -c 600 gpurun_out/bench139.txt
