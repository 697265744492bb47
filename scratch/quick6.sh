#!/bin/bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/q_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/q_pytest.log
tail -3 gpurun_out/q_pytest.log
for v in 1 0; do
APT_FUSED_OUT=$v timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 50 > gpurun_out/q_bench_fo$v.log 2>&1
tail -1 gpurun_out/q_bench_fo$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('fused_out=$v', d['ms_per_step'], d['phases_ms'])"
done
