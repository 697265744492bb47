#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$? $(tail -1 gpurun_out/q_pytest.log)"
grep -E "FAIL|Error" gpurun_out/q_pytest.log | head -5
for rep in 1 2; do
for v in 0 1; do
  APT_SAMPLE_G16=$v timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_g.log 2>&1
  tail -1 gpurun_out/ab_g.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('g16=$v', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/q_launches_g16.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-planner --no-pipeline > /dev/null 2>&1
