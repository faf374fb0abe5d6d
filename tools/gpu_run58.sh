nvidia-smi -q -d POWER > gpurun_out/power58.txt 2>&1
(echo "# compute-sanitizer (round 1, after the warp-uniform MMA change) on tools/sanitize_cases.py: f32, bf16 resident, bf16 streaming 1-CTA / CTA-pair / 32-unit tiles, dilated, grid (bf16 + f32), layer-sequential, linear RNN, b2b GEMM"
echo "## memcheck"; timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_cases.py 2>&1 | tail -3
echo "## synccheck"; timeout 900 compute-sanitizer --tool synccheck python tools/sanitize_cases.py 2>&1 | tail -3
echo "## racecheck"; timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_cases.py 2>&1 | tail -3) > gpurun_out/sanitizer58.txt
