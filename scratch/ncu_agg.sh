#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'agg_l1' --launch-skip 3 -c 2 -o gpurun_out/agg_full \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-planner > gpurun_out/agg_full.log 2>&1
echo done
