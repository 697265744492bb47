#!/bin/bash
# Round evidence on one B200 (run from the repo root under gpurun): GPU tests, smoke, the
# bench line, the reference (oracle) arm, the ncu launch list of the bench command and
# `ncu --set full` captures of the dominant kernel and the step's main-chain kernels.
# Writes gpurun_out/final_*.
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/final_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/final_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/final_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final_launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'agg_l1' --launch-skip 3 -c 2 \
  -o gpurun_out/final_agg_full python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-planner \
  > gpurun_out/final_agg_full.log 2>&1
bash tools/ncu_step.sh final_step
