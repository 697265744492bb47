#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/f3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f3_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/f3_smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/f3_bench.log 2>&1
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f3_launches.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner > /dev/null 2>&1
