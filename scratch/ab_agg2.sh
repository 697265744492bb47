#!/bin/bash
# A/B: layer-1 gather+mean with 5 loads in flight (variants 6/7) and the grid cap per SM.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ab2_build.log 2>&1
for v in 7; do
  APT_AGG_VARIANT=$v timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/ab2_pytest$v.log 2>&1; echo "variant $v pytest rc=$? $(tail -1 gpurun_out/ab2_pytest$v.log)"
done
APT_AGG_VARIANT=7 APT_AGG_BPSM=4 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/ab2_pytest_b5.log 2>&1; echo "bpsm 5 pytest rc=$? $(tail -1 gpurun_out/ab2_pytest_b5.log)"
for rep in 1 2; do
for cfg in "5 5" "5 4" "5 3" "7 4" "7 8" "7 16"; do
  set -- $cfg
  APT_AGG_VARIANT=$1 APT_AGG_BPSM=$2 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/ab2_$1_$2.log 2>&1
  tail -1 gpurun_out/ab2_$1_$2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('variant $1 bpsm $2', round(d['ms_per_step'],4), 'agg', round(d['phases_ms'].get('agg_kernel',-1),4), 'frac', round(d['roofline']['frac'],3))"
done
done
