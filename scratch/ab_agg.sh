#!/bin/bash
set -u
mkdir -p gpurun_out
for v in 4 5; do
  APT_AGG_VARIANT=$v timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/ab_agg_pytest$v.log 2>&1; echo "variant $v pytest rc=$? $(tail -1 gpurun_out/ab_agg_pytest$v.log)"
done
for rep in 1 2; do
for v in 1 4 5; do
  APT_AGG_VARIANT=$v timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab_agg$v.log 2>&1
  tail -1 gpurun_out/ab_agg$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('variant $v', round(d['ms_per_step'],4), 'agg', round(d['phases_ms']['agg_kernel'],4), 'frac', round(d['roofline']['frac'],3))"
done
done
