# compute-sanitizer (memcheck, synccheck, racecheck) on every kernel variant, incl. the round-2b features
python tools/sanitize_cases.py > gpurun_out/san144_plain.txt 2>&1
timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > gpurun_out/san144.txt 2>&1
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_cases.py >> gpurun_out/san144.txt 2>&1
timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_cases.py >> gpurun_out/san144.txt 2>&1
tail -2 gpurun_out/san144_plain.txt; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|done" gpurun_out/san144.txt
