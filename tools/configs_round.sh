#!/bin/bash
# Round-end config evidence on one B200 (run under gpurun, after tools/profile_round.sh or
# alone): BASELINE configs 1-5 (tools/round_configs.sh), the fp32 products bench line and
# the Fig. 8c cache sweeps.  Writes gpurun_out/cfg_* and gpurun_out/sweep_*.
set -u
mkdir -p gpurun_out
timeout 600 python bench.py --dtype f32 --steps 100 --warmup 20 > gpurun_out/cfg_products_f32.json 2> gpurun_out/cfg_f32.err
bash tools/round_configs.sh
timeout 2400 python tools/sweep.py products-cache > gpurun_out/sweep_products_cache.jsonl 2> gpurun_out/sweep_products_cache.err
timeout 3000 python tools/sweep.py friendster-cache > gpurun_out/sweep_friendster_cache.jsonl 2> gpurun_out/sweep_friendster_cache.err
