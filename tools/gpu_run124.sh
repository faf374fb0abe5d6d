# round-end style validation: full GPU suite, smoke, bench (1 GPU), 2-rank path (gloo control plane, one GPU)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest124.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke124.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench124.txt 2>&1
FT_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench124_2rank.txt 2>&1
FT_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --gpus 2 --steps 10 --warmup 3 --no-cpu-baseline --gather fused > gpurun_out/bench124_2rank_fused.txt 2>&1
