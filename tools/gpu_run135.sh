timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "c_abi_example" > gpurun_out/pytest135.txt 2>&1
gcc -O2 -I include -I /usr/local/cuda/include examples/c_abi_example.c -L paper_conf_sosp_liuqc0hs0y24_b200 -lft -L /usr/local/cuda/lib64 -lcudart -lm -Wl,-rpath,$PWD/paper_conf_sosp_liuqc0hs0y24_b200 -o /tmp/cex && /tmp/cex > gpurun_out/c_example135.txt 2>&1
