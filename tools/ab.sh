#!/bin/bash
# A/B of environment knobs on the products bench step (run under gpurun):
#   tools/ab.sh "ENV=1 ENV2=3" "ENV=0" ...   (each argument one configuration; "" = defaults)
mkdir -p gpurun_out
for cfg in "$@"; do
  for rep in 1 2; do
    env $cfg timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 60 --warmup 10 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms']; print('[$cfg] rep $rep', round(d['ms_per_step'],4), 'l1', round(p['layer1_fwd']*1e3,1), 'agg', round(p['agg_kernel']*1e3,1), 'up', round(p['upper_fwd_loss']*1e3,1), 'bwd', round(p['backward']*1e3,1), 'sgd', round(p['allreduce_sgd']*1e3,1))"
  done
done
