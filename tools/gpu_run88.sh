# compute-sanitizer after the round-2 kernel changes (coalesced c ring, 256-bit h stores, persisting window)
echo "## memcheck" > gpurun_out/san88.txt
timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_cases.py >> gpurun_out/san88.txt 2>&1
echo "## synccheck" >> gpurun_out/san88.txt
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_cases.py >> gpurun_out/san88.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest88.txt 2>&1
