#!/bin/bash
# BASELINE configs 1-5 on one B200 (run under gpurun): bench lines of tiny and the GAT model,
# the papers d sweep and the friendster hidden sweep (measured C = 1 step, Planner
# predictions at C = 2/4/8 from full-epoch dry runs, every strategy emulated at C <= 4).
mkdir -p gpurun_out
timeout 600 python bench.py --config tiny --steps 100 --warmup 20 > gpurun_out/cfg_tiny.json 2> gpurun_out/cfg_tiny.err
timeout 900 python bench.py --gat-heads 4 --steps 50 --warmup 10 > gpurun_out/cfg_products_gat4.json 2> gpurun_out/cfg_gat.err
timeout 2400 python tools/sweep.py papers-d --dryrun-steps 0 > gpurun_out/cfg_papers_d.jsonl 2> gpurun_out/cfg_papers.err
timeout 2400 python tools/sweep.py friendster-h --dryrun-steps 0 > gpurun_out/cfg_friendster_h.jsonl 2> gpurun_out/cfg_friendster.err
timeout 1800 python tools/sweep.py papers-gat --dryrun-steps 16 > gpurun_out/cfg_papers_gat.jsonl 2> gpurun_out/cfg_papers_gat.err
