#!/bin/bash
set -u
mkdir -p gpurun_out
for rep in 1 2; do
for cfg in "0 4" "1 4" "0 3" "0 6"; do
set -- $cfg
  APT_FUSED_OUT=$1 APT_BG_BLOCKS_PER_SM=$2 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_m.log 2>&1
  tail -1 gpurun_out/ab_m.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('fused_out=$1 bg=$2', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
