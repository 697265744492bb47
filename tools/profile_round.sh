#!/bin/bash
# Round evidence on one B200 (run from the repo root under gpurun): GPU tests, the bench
# line, the reference (oracle) arm, the ncu launch list of the bench command and one
# `ncu --set full` capture of the step's top kernels.  Writes gpurun_out/final_*.
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/final_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/final_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/final_smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/final_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.log 2>&1
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final_launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:'agg_l1|rowtile_kernel|pull_bwd_kernel|wgrad_kernel|sample_kernel|compact_scan|outlayer_kernel|agg_kernel' \
  --launch-skip 40 -c 24 -o gpurun_out/final_full python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-planner \
  > gpurun_out/final_ncu_full.log 2>&1
