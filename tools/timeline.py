"""Kernel timeline of the pipelined bench step (CUPTI through torch.profiler; no nsys here).

Builds the bench's products trainer, warms up, then records a few steps exactly as bench.py
times them (L2 flush, graph replay, sync) and prints, for one step, every kernel with its
start offset from the step's first kernel, its duration and its stream, so the overlap of
the main chain and the next step's sampling branch can be read off.

    python tools/timeline.py [--config products] [--steps 4] [--out gpurun_out/timeline.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="products")
    ap.add_argument("--steps", type=int, default=4)
    ap.add_argument("--dtype", default="bf16")
    ap.add_argument("--out", default="gpurun_out/timeline.json")
    ap.add_argument("--no-pipeline", action="store_true")
    ap.add_argument("--sync-flush", action="store_true",
                    help="synchronize between the L2 flush and the step (exposes the host graph launch); "
                         "default: like bench.py, the launch overlaps the flush")
    args = ap.parse_args()
    import torch
    from torch.profiler import ProfilerActivity, profile

    import aptgen
    import bench
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A

    bench.GAT_HEADS = 0
    cfg = aptgen.CONFIGS[args.config]
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(priority=-1)
    torch.cuda.set_stream(stream)
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    ctx = A.Ctx(0, 1, 0, stream.cuda_stream)
    gr = ctx.graph_load(g.indptr, g.indices, None)
    fs = ctx.fstore_create(gr, A.GDP, A.DTYPE[args.dtype], cfg.dim, None, cfg.feat_seed)
    tr = bench.make_trainer(A, ctx, gr, fs, cfg, A.DTYPE[args.dtype], A.GDP, labels)
    tr.set_params(aptgen.weights(cfg))
    tr.set_epoch(train, 0)
    tr.use_graph(True)
    if args.no_pipeline:
        tr.set_pipeline(False)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    flush_rd = torch.ones(64 << 20, dtype=torch.int32, device="cuda")   # bench.py --flush write+read
    flush_out = torch.empty((), dtype=torch.int32, device="cuda")
    for i in range(10):
        tr.step(i)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for i in range(args.steps):
            flush.zero_()
            torch.amax(flush_rd, dim=0, out=flush_out)
            if args.sync_flush:
                torch.cuda.synchronize()
            tr.step(10 + i)
            torch.cuda.synchronize()
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    prof.export_chrome_trace(args.out)
    ev = [e for e in json.load(open(args.out))["traceEvents"] if e.get("cat") == "kernel"]
    ev.sort(key=lambda e: e["ts"])
    # split into steps at the flush kernels (FillFunctor / zero_)
    steps, cur, fl_end = [], None, []
    for e in ev:
        if "FillFunctor" in e["name"]:
            cur = []
            steps.append(cur)
            fl_end.append(e["ts"] + e["dur"])
        elif cur is not None and not cur and "reduce_kernel" in e["name"]:   # the flush's read pass
            fl_end[-1] = e["ts"] + e["dur"]
        elif cur is not None:
            cur.append(e)
    for si, st in enumerate(steps[1:3], 1):
        if not st:
            continue
        t0 = st[0]["ts"]
        t1 = max(e["ts"] + e["dur"] for e in st)
        print(f"# step {si}: {len(st)} kernels, first->last end {t1 - t0:.1f} us; "
              f"L2 flush end -> first kernel {t0 - fl_end[si]:.1f} us")
        streams = sorted({e["args"].get("stream", 0) for e in st})
        for e in st:
            s = e["args"].get("stream", 0)
            col = streams.index(s)
            name = e["name"].replace("void ", "").replace("apt::", "")[:60]
            print(f"{e['ts'] - t0:8.1f} {e['dur']:7.1f}  s{col} {'    ' * col}{name}")


if __name__ == "__main__":
    main()
