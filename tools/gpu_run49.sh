python -m paper_conf_sosp_liuqc0hs0y24_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "layerwise" -m "gpu" > gpurun_out/lw_tests.txt 2>&1
timeout 600 python tools/layerwise_time.py > gpurun_out/lw_time.jsonl 2>&1
