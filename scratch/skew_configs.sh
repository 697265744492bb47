#!/bin/bash
# papers / friendster bench lines with the planner (access-skew table vs Table 3)
set -u
mkdir -p gpurun_out
for c in papers friendster; do
  SECONDS=0; timeout 1500 python bench.py --config $c --steps 50 --warmup 10 --no-cpu-baseline --emulate-max-c 0 > gpurun_out/skew_$c.log 2> gpurun_out/skew_$c.err
  echo "$c wall $SECONDS s"; tail -2 gpurun_out/skew_$c.err
  tail -1 gpurun_out/skew_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['ms_per_step'], d['access_skew']['table'], d['step_roofline']['frac'], d['roofline']['frac'])"
done
