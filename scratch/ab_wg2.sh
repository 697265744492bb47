#!/bin/bash
set -u
mkdir -p gpurun_out
for rep in 1 2; do
for cfg in "1 3" "2 3" "1 6" "2 6"; do
set -- $cfg
  APT_WG_SPLITS_PER_SM=$1 APT_WG_STAGES=$2 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_w2.log 2>&1
  tail -1 gpurun_out/ab_w2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('splits/sm=$1 stages=$2', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
