./build/smem_base > gpurun_out/smem_base.txt 2>&1
