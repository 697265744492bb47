#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$? $(tail -1 gpurun_out/q_pytest.log)"
for rep in 1 2; do
for v in 0 1; do
  APT_CSC_COUNT_IN_MAP=$v timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_cim.log 2>&1
  tail -1 gpurun_out/ab_cim.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('count_in_map=$v', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
