#!/usr/bin/env bash
# Same-box A/B of environment settings through bench.py (device-timed C3 step, the bench regime):
#   bash tools/ab_env.sh TAG REPS "ENV1" "ENV2" ...   (an ENV is "" for the default or "K=V K2=V2")
TAG=$1; REPS=$2; shift 2
mkdir -p gpurun_out
f=gpurun_out/${TAG}_abenv.txt
for i in $(seq 1 "$REPS"); do
  for e in "$@"; do
    env $e timeout 600 python bench.py --steps ${AB_STEPS:-20} --warmup 5 --no-cpu-baseline --no-parity 2>/dev/null | grep '^{' | \
      python -c "import sys,json; d=json.loads(sys.stdin.read()); c=d['clocks'] or {}; print('[$e]', round(d['ms_per_step'],3), round(d['value']), round(d['roofline']['frac'],3), c.get('sm_mhz'), c.get('power_w_median'), c.get('reasons'), round(d['e2e']['value']))" >> "$f"
  done
done
cat "$f"
