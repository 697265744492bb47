#!/bin/bash
# refresh the non-default bench lines (GAT products, papers, friendster, tiny) at the round's final code
set -u
mkdir -p gpurun_out
timeout 900 python bench.py --gat-heads 4 --cpu-steps 1 --emulate-max-c 2 > gpurun_out/line_gat4.log 2> gpurun_out/line_gat4.err; echo "gat rc=$?"
timeout 900 python bench.py --config tiny --emulate-max-c 4 > gpurun_out/line_tiny.log 2> gpurun_out/line_tiny.err; echo "tiny rc=$?"
for c in papers friendster; do
  timeout 1500 python bench.py --config $c --steps 50 --warmup 10 --no-cpu-baseline --emulate-max-c 0 > gpurun_out/line_$c.log 2> gpurun_out/line_$c.err; echo "$c rc=$?"
done
