timeout 120 ./build/umma_bench > gpurun_out/umma_bench.txt 2>&1
