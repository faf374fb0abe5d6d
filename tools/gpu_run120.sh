for i in 1 2; do timeout 600 python bench.py > gpurun_out/bench120_$i.txt 2>&1; done
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench120_ref.txt 2>&1
