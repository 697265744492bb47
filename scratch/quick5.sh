#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_access.py -m gpu -x -q > gpurun_out/q_pytest_access.log 2>&1; echo "rc=$?" >> gpurun_out/q_pytest_access.log
tail -2 gpurun_out/q_pytest_access.log
timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 50 --no-pipeline > gpurun_out/q_bench_nopipe.log 2>&1
tail -1 gpurun_out/q_bench_nopipe.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('nopipe', d['ms_per_step'], d['phases_ms'])"
timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 50 > gpurun_out/q_bench.log 2>&1
tail -1 gpurun_out/q_bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('pipe', d['ms_per_step'], d['phases_ms'])"
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/q_launches_warm.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner --no-pipeline > /dev/null 2>&1
