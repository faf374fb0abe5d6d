#!/usr/bin/env bash
# One parameterised GPU runner (replaces round 1's one-off tools/gpu_run*.sh scripts).
#
#   gpurun --timeout 1800 -- 'bash tools/gpu.sh TAG step [step ...]'
#
# Every step writes gpurun_out/<TAG>_<step>.txt and prints its tail.  Steps:
#   suite            python -m pytest tests -m gpu -q            (full GPU suite)
#   pytest:EXPR      python -m pytest tests -m gpu -q -k EXPR      (subset)
#   smoke            __graft_entry__.smoke()
#   bench            python bench.py (defaults; N=1 with the CPU baseline)
#   benchq           python bench.py --no-cpu-baseline (x2, same box)
#   bench2 / bench4  bench.py --gpus N with N ranks sharing cuda:0 (gloo control plane, fused gather)
#   qt:CFGS          tools/quick_time.py CFGS (comma separated, e.g. qt:C2,C3,C4,C5)
#   launches         ncu launch list of a short bench run (gpu__time_duration, no clock control)
#   ncu:CFG          ncu --set full of the first wavefront launch of tools/quick_time.py CFG
#   sanitize         tools/sanitize_cases.py under compute-sanitizer
#   ab:LIBS:CFGS     same-box A/B: for each build/ab/libft_<lib>.so, 3 interleaved quick_time runs
# Environment: QT_REPS (default 30) is passed through to quick_time.
set -u
TAG=$1; shift
mkdir -p gpurun_out
out() { echo "gpurun_out/${TAG}_$1.txt"; }
for step in "$@"; do
  case "$step" in
    suite)   timeout 1800 python -m pytest tests -m gpu -q > "$(out suite)" 2>&1; tail -3 "$(out suite)";;
    pytest:*) k=${step#pytest:}; f=$(out "pytest_${k//[^A-Za-z0-9]/_}")
             timeout 1500 python -m pytest tests -m gpu -q -k "$k" > "$f" 2>&1; tail -3 "$f";;
    smoke)   timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > "$(out smoke)" 2>&1; tail -1 "$(out smoke)";;
    bench)   timeout 900 python bench.py > "$(out bench)" 2>&1; tail -c 600 "$(out bench)"; echo;;
    benchq)  for i in 1 2; do timeout 600 python bench.py --no-cpu-baseline >> "$(out benchq)" 2>&1; done
             grep '^{' "$(out benchq)" | python -c "import sys,json
for l in sys.stdin:
    d=json.loads(l); print(round(d['ms_per_step'],3), round(d['value']), d['roofline']['frac'], d['clocks'] and d['clocks']['sm_mhz'], d['e2e']['value'])";;
    bench2|bench4) n=${step#bench}
             FT_BENCH_SHARED_GPU=1 FT_DIST_BACKEND=gloo timeout 900 python bench.py --gpus "$n" --steps 4 --warmup 3 --no-cpu-baseline > "$(out "$step")" 2>&1
             tail -c 800 "$(out "$step")"; echo;;
    qt:*)    cf=${step#qt:}; QT_REPS=${QT_REPS:-30} timeout 900 python tools/quick_time.py ${cf//,/ } > "$(out "qt_${cf//,/_}")" 2>&1; cat "$(out "qt_${cf//,/_}")";;
    launches) timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
               --log-file "gpurun_out/${TAG}_launches.csv" python bench.py --steps 5 --warmup 3 --no-cpu-baseline > "$(out launches)" 2>&1
             tail -2 "$(out launches)";;
    ncu:*)   cf=${step#ncu:}
             timeout 1200 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 \
               -o "gpurun_out/${TAG}_${cf}" python tools/quick_time.py "$cf" > "$(out "ncu_$cf")" 2>&1
             tail -2 "$(out "ncu_$cf")";;
    sanitize) timeout 1500 python tools/sanitize_cases.py > "$(out sanitize)" 2>&1; tail -20 "$(out sanitize)";;
    ab:*)    rest=${step#ab:}; libs=${rest%%:*}; cfgs=${rest#*:}
             f=$(out "ab_${libs//,/_}")
             for i in 1 2 3; do for v in ${libs//,/ }; do
               FT_LIB_PATH=build/ab/libft_$v.so QT_REPS=${QT_REPS:-30} timeout 600 python tools/quick_time.py ${cfgs//,/ } 2>&1 | sed "s/^/$v /" >> "$f"
             done; done; cat "$f";;
    dram:*)  rest=${step#dram:}; lib=${rest%%:*}; cf=${rest#*:}; f=$(out "dram_${lib}_${cf}")
             FT_LIB_PATH=build/ab/libft_$lib.so QT_REPS=3 QT_WARM=2 timeout 300 ncu --metrics \
               gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
               --clock-control none -k regex:wavefront -s 2 -c 1 --csv python tools/quick_time.py "$cf" > "$f" 2>&1
             grep -E "dram__|gpu__time|lts__t_bytes|tensor_cycles" "$f" | awk -F'","' '{print $(NF-2), $(NF-1), $NF}';;
    *) echo "unknown step $step";;
  esac
done
