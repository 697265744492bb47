#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/q_pytest.log
tail -3 gpurun_out/q_pytest.log
timeout 600 python bench.py --no-planner --no-cpu-baseline --steps 50 > gpurun_out/q_bench.log 2>&1
tail -1 gpurun_out/q_bench.log | cut -c1-300
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/rt_lat.csv python scratch/rowtile_lat.py > gpurun_out/rt_lat.log 2>&1
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/q_launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner > /dev/null 2>&1
