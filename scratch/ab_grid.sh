#!/bin/bash
# A/B: grid caps (blocks per SM) of the upper-layer mean and the bf16 mean backward.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/abg_build.log 2>&1
APT_AGGU_BPSM=4 APT_PULL_BPSM=4 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/abg_pytest.log 2>&1; echo "caps 4/4 pytest rc=$? $(tail -1 gpurun_out/abg_pytest.log)"
for rep in 1 2; do
for cfg in "16 16" "6 16" "4 16" "16 8" "16 4" "6 8"; do
  set -- $cfg
  APT_AGGU_BPSM=$1 APT_PULL_BPSM=$2 timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 100 > gpurun_out/abg_$1_$2.log 2>&1
  tail -1 gpurun_out/abg_$1_$2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('aggu $1 pull $2', round(d['ms_per_step'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
