# compute-sanitizer on every kernel variant incl. layer bands (owner / round-robin, skew 2)
timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > gpurun_out/san112.txt 2>&1
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_cases.py >> gpurun_out/san112.txt 2>&1
timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_cases.py >> gpurun_out/san112.txt 2>&1
