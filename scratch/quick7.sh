#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/q_launches_fo.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner --no-pipeline > /dev/null 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:outlayer --launch-skip 3 -c 1 -o gpurun_out/q_outlayer \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner --no-pipeline > /dev/null 2>&1
APT_FUSED_OUT=1 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 50 --no-pipeline > gpurun_out/q_bench_fo1_np.log 2>&1
tail -1 gpurun_out/q_bench_fo1_np.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('fo1 nopipe', d['ms_per_step'], d['phases_ms'])"
