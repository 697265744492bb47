"""Parameter sweeps of BASELINE configs 3-5 and the fanout sweep
on one B200: the graph is generated once per config, then for every variant one JSON
line with the measured 1-GPU step (GDP, CUDA graph, L2 flushed), the Planner's Eq. 2
prediction per strategy at C = 2, 4, 8 and every strategy's step with C ranks emulated
on this GPU (C <= --emulate-max-c).  Uses bench.py's trainer / planner code.

  python tools/sweep.py papers-d         # config 3: papers, d in {64, 256}
  python tools/sweep.py friendster-h     # config 4: friendster d=256, hidden {8, 32, 128}
  python tools/sweep.py papers-gat       # config 5: papers d=128, GAT 4 heads, hidden 32..1024
  python tools/sweep.py products-fanout  # fanouts [10,5], [15,10], [20,15,10]
  python tools/sweep.py products-cache   # Fig. 8c: P:163 GPU cache size sweep, C = 4
  python tools/sweep.py friendster-cache # the same on the friendster shape (FS skew)
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
    # Fig. 8c: per-GPU cache budget (fraction of the nodes) under P:163's rules
    "products-cache": ("products", [dict(cache=f) for f in (0.0, 0.01, 0.05, 0.1, 0.25, 0.5)], 0),
    "papers-cache": ("papers", [dict(cache=f) for f in (0.0, 0.01, 0.05, 0.1, 0.25)], 0),
    "friendster-cache": ("friendster", [dict(cache=f) for f in (0.0, 0.01, 0.05, 0.1, 0.25)], 0),
}


def cache_point(A, g, cfg, train, labels, stream, dt, frac, counts, C=4, steps=5, dryrun_steps=0):
    """One point of Fig. 8c: for GDP, SNP and DNP a store of P:163 caches of frac * n rows per
    GPU (APT_CACHE_P163: own cache, else a peer's over NVLink, else the pinned host), the
    strategy's full step with C ranks emulated on this GPU (ms, 5 steps after 3) and the
    Planner's Eq. 2 prediction for that strategy from a dry run on the same store.  NFP
    keeps its 1/C column slice of every row and is reported once, as is."""
    out = {}
    budget = int(frac * g.n)
    part = bench.partition(A, g, C)
    for s in ("GDP", "NFP", "SNP", "DNP"):
        ctx = A.Ctx(-1, C, 0, stream.cuda_stream)
        gr = ctx.graph_load(g.indptr, g.indices, part)
        if s == "NFP":
            fs = ctx.fstore_create(gr, A.NFP, dt, cfg.dim, None, cfg.feat_seed)
        else:
            fs = ctx.fstore_create(gr, A.STRATEGY[s], dt, cfg.dim, None, cfg.feat_seed, counts=counts,
                                   cache_budget_rows=budget)
        tr = bench.make_trainer(A, ctx, gr, fs, cfg, dt, A.STRATEGY[s], labels)
        tr.set_params(aptgen.weights(cfg))
        tr.set_epoch(train, 0)
        st = tr.dryrun(dryrun_steps or tr.steps_per_epoch())
        bw = ctx.profile_links()
        pick, pred = A.select_strategy(st, bw)
        si = bench.STRATS.index(s)
        nst = max(1, st.steps)
        tr.use_graph(True)
        for i in range(3):
            tr.step(i)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(3, 3 + steps):
            tr.step(i)
        e1.record(stream)
        torch.cuda.synchronize()
        out[s] = {"emulated_ms_per_step": e0.elapsed_time(e1) / steps,
                  "pred_ms_per_step": 1e3 * pred[si] / nst,
                  "rows_local_per_step": sum(st.rows_local[si][r] for r in range(C)) / nst,
                  "rows_peer_per_step": sum(st.rows_peer[si][r] for r in range(C)) / nst,
                  "rows_host_per_step": sum(st.rows_host[si][r] for r in range(C)) / nst}
        for h in (tr, fs, gr):
            h.close()
        ctx.close()
        torch.cuda.empty_cache()
    out["pred_pick"] = min(("GDP", "NFP", "SNP", "DNP"), key=lambda k: out[k]["pred_ms_per_step"])
    out["emulated_fastest"] = min(("GDP", "NFP", "SNP", "DNP"), key=lambda k: out[k]["emulated_ms_per_step"])
    return out


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
    counts = None
    for v in variants:
        v = dict(v)
        if "cache" in v:   # Fig. 8c: access counts of one epoch (C = 4, GDP split), then every budget
            frac = v["cache"]
            cfg = base
            rec = {"sweep": args.sweep, "variant": v, "config": bench.workload_config(cfg), "dtype": args.dtype,
                   "C": 4, "cache_rows_per_gpu": int(frac * g.n), "graph_gen_s": round(t_gen, 1)}
            try:
                if counts is None:
                    ctx = A.Ctx(-1, 4, 0, stream.cuda_stream)
                    gr = ctx.graph_load(g.indptr, g.indices, bench.partition(A, g, 4))
                    fs = ctx.fstore_create(gr, A.GDP, dt, cfg.dim, None, cfg.feat_seed)
                    tr = bench.make_trainer(A, ctx, gr, fs, cfg, dt, A.GDP, labels)
                    tr.set_epoch(train, 0)
                    counts = tr.access_counts(tr.steps_per_epoch())
                    for h in (tr, fs, gr):
                        h.close()
                    ctx.close()
                rec["strategies"] = cache_point(A, g, cfg, train, labels, stream, dt, frac, counts,
                                                dryrun_steps=args.dryrun_steps)
            except Exception as e:
                rec["error"] = repr(e)[:400]
            print(json.dumps(rec), flush=True)
            torch.cuda.empty_cache()
            continue
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
