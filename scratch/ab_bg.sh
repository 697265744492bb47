#!/bin/bash
set -u
mkdir -p gpurun_out
for rep in 1 2; do
for cfg in "4 0" "2 0" "1 0" "8 0" "4 1" "2 1"; do
set -- $cfg
  APT_BG_BLOCKS_PER_SM=$1 APT_SAMPLE_FORK=$2 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_bg.log 2>&1
  tail -1 gpurun_out/ab_bg.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bg=$1 fork=$2', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
