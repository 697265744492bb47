"""Parameter sweeps of BASELINE configs 3-5 and the fanout sweep
on one B200: the graph is generated once per config, then for every variant one JSON
line with the measured 1-GPU step (GDP, CUDA graph, L2 flushed), the Planner's Eq. 2
prediction per strategy at C = 2, 4, 8 and every strategy's step with C ranks emulated
on this GPU (C <= --emulate-max-c).  Uses bench.py's trainer / planner code.

  python tools/sweep.py papers-d         # config 3: papers, d in {64, 256}
  python tools/sweep.py friendster-h     # config 4: friendster d=256, hidden {8, 32, 128}
  python tools/sweep.py papers-gat       # config 5: papers d=128, GAT 4 heads, hidden 32..1024
  python tools/sweep.py products-fanout  # fanouts [10,5], [15,10], [20,15,10]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import aptgen  # noqa: E402
import bench  # noqa: E402

SWEEPS = {
    "papers-d": ("papers", [dict(dim=64), dict(dim=256)], 0),
    "friendster-h": ("friendster", [dict(hidden=8), dict(hidden=32), dict(hidden=128)], 0),
    "papers-gat": ("papers", [dict(dim=128, hidden=h) for h in (32, 128, 512, 1024)], 4),
    "products-fanout": ("products", [dict(fanouts=(10, 5)), dict(fanouts=(15, 10)), dict(fanouts=(20, 15, 10))], 0),
    "papers-gat-wide": ("papers", [dict(dim=128, hidden=1024)], 4),
    "tiny-gat": ("tiny", [dict(hidden=32), dict(hidden=128)], 4),
    # Fig. 11 partition-quality ablation: planted range vs random vs LDG streaming
    "products-partition": ("products", [dict(partition=p) for p in ("range", "random", "ldg")], 0),
    "papers-partition": ("papers", [dict(partition=p) for p in ("range", "random", "ldg")], 0),
}


def measure_gdp(A, g, cfg, train, labels, stream, dt, steps=20, warmup=5):
    ctx = A.Ctx(0, 1, 0, stream.cuda_stream)
    gr = ctx.graph_load(g.indptr, g.indices, aptgen.partition(g.n, 1))
    fs = ctx.fstore_create(gr, A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    tr = bench.make_trainer(A, ctx, gr, fs, cfg, dt, A.GDP, labels)
    tr.set_params(aptgen.weights(cfg))
    tr.set_epoch(train, 0)
    tr.use_graph(True)
    spe = tr.steps_per_epoch()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for i in range(warmup):
        tr.step(i % spe)
    torch.cuda.synchronize()
    ms, l1 = [], []
    for i in range(steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        tr.step((warmup + i) % spe)
        e1.record(stream)
        ph = tr.phase_ms()
        ms.append(e0.elapsed_time(e1))
        l1.append(ph[5])
    out = {"ms_per_step": float(np.mean(ms)), "seeds_per_s": cfg.batch / (np.mean(ms) / 1e3),
           "layer1_kernel_ms": float(np.mean(l1)), "steps_per_epoch": spe,
           "epoch_s": spe * float(np.mean(ms)) / 1e3}
    for h in (tr, fs, gr):
        h.close()
    ctx.close()
    del flush
    torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("sweep", choices=sorted(SWEEPS))
    ap.add_argument("--dtype", default="bf16")
    ap.add_argument("--dryrun-steps", type=int, default=8)
    ap.add_argument("--emulate-max-c", type=int, default=4)
    args = ap.parse_args()
    name, variants, heads = SWEEPS[args.sweep]
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(priority=-1)
    torch.cuda.set_stream(stream)
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    A.lib()
    base = aptgen.CONFIGS[name]
    t0 = time.time()
    g = aptgen.make_graph(base)
    t_gen = time.time() - t0
    train = aptgen.train_nodes(g, base)
    labels = aptgen.labels(base, g.n)
    bench.GAT_HEADS = heads
    dt = A.DTYPE[args.dtype]
    for v in variants:
        v = dict(v)
        bench.PARTITION = v.pop("partition", "range")
        cfg = base.replace(**v)
        if bench.PARTITION != "range":
            v["partition"] = bench.PARTITION
        rec = {"sweep": args.sweep, "variant": {k: list(x) if isinstance(x, tuple) else x for k, x in v.items()},
               "config": bench.workload_config(cfg), "dtype": args.dtype, "gat_heads": heads,
               "graph_gen_s": round(t_gen, 1)}
        try:
            rec["measured_c1_gdp"] = measure_gdp(A, g, cfg, train, labels, stream, dt)
            ns = argparse.Namespace(dtype=args.dtype, dryrun_steps=args.dryrun_steps, emulate_max_c=args.emulate_max_c)
            rec["planner"] = bench.planner_report(A, g, cfg, train, labels, ns, stream,
                                                  rec["measured_c1_gdp"]["ms_per_step"])
        except Exception as e:   # report and continue with the next variant
            rec["error"] = repr(e)[:400]
        print(json.dumps(rec), flush=True)
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
