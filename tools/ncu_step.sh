#!/bin/bash
# ncu --set full of one bench step's main-chain kernels (layer-1 gather, every projection,
# weight gradient and mean backward), skipping the warm-up steps.  Run under gpurun.
#   tools/ncu_step.sh <tag> [bench args...]
set -u
tag=$1; shift
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:'rowtile_kernel|wgrad_kernel|pull_bwd|agg_l1|agg_kernel|ce_loss' --launch-skip 39 -c 13 \
  -o gpurun_out/${tag} python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-planner "$@" \
  > gpurun_out/${tag}.log 2>&1
bash tools/ncu_summary.sh gpurun_out/${tag}.ncu-rep > gpurun_out/${tag}_summary.csv
