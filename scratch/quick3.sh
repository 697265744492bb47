#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/rt_lat.csv python scratch/rowtile_lat.py > gpurun_out/rt_lat.log 2>&1
timeout 300 python scratch/gather_ceiling.py > gpurun_out/gather_ceiling.log 2>&1
for v in 1 2 4; do
  APT_PROJ_SPLIT=$v timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 50 > gpurun_out/ab_split$v.log 2>&1
  echo "split $v: $(tail -1 gpurun_out/ab_split$v.log | cut -c1-200)"
done
