#!/usr/bin/env bash
# Same-box A/B of library builds through bench.py (device value and e2e):
#   bash tools/ab_lib_bench.sh TAG REPS lib1 lib2 ...   (build/ab/libft_<lib>.so)
TAG=$1; REPS=$2; shift 2
mkdir -p gpurun_out
f=gpurun_out/${TAG}_ablib.txt
for i in $(seq 1 "$REPS"); do
  for v in "$@"; do
    FT_LIB_PATH=build/ab/libft_$v.so timeout 600 python bench.py --steps ${AB_STEPS:-20} --warmup 5 --no-cpu-baseline --no-parity 2>/dev/null | grep '^{' | \
      python -c "import sys,json; d=json.loads(sys.stdin.read()); c=d['clocks'] or {}; print('$v', round(d['ms_per_step'],3), round(d['value']), 'e2e', round(d['e2e']['value']), d['e2e']['matches_device_path'], c.get('sm_mhz'))" >> "$f"
  done
done
cat "$f"
