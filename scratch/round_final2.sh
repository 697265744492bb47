#!/bin/bash
set -u
bash scratch/profile_round.sh
bash scratch/ncu_agg.sh
timeout 900 python bench.py --config papers --steps 50 --warmup 10 --no-cpu-baseline --emulate-max-c 0 > gpurun_out/line_papers.log 2> gpurun_out/line_papers.err; echo "papers rc=$?"
