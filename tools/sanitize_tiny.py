"""The tiny config under compute-sanitizer: one training step of every
strategy (C = 1 GDP in f32 and bf16, C = 2 emulated NFP / SNP / DNP in bf16, a GAT
layer 1), the standalone layer API, and the tensor-core GEMM / sort self-tests.
  compute-sanitizer --tool memcheck  python tools/sanitize_tiny.py
  compute-sanitizer --tool racecheck python tools/sanitize_tiny.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import aptgen  # noqa: E402
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A  # noqa: E402


def main():
    torch.cuda.set_device(0)
    cfg = aptgen.CONFIGS["tiny"]
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    base = cfg
    # (the last run: the tiny graph under the benchmark's model shape -- 3 layers, hidden
    # 256 -- so the 128-column projection slices take the TMA-store epilogue)
    runs = [("GDP", 1, "f32", 0, None), ("GDP", 1, "bf16", 0, None), ("NFP", 2, "bf16", 0, None),
            ("SNP", 2, "bf16", 0, None), ("DNP", 2, "bf16", 0, None), ("DNP", 2, "f32", 4, None),
            ("GDP", 1, "bf16", 0, dict(hidden=256, fanouts=(5, 5, 5)))]
    for strategy, C, dtype, heads, var in runs:
        cfg = base.replace(**var) if var else base
        dims = [cfg.dim] + [d for _, d in cfg.dims()]
        ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
        gr = ctx.graph_load(g.indptr, g.indices, aptgen.partition(g.n, C))
        dt = A.DTYPE[dtype]
        fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
        tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, 0.1, cfg.sample_seed, cfg.feat_seed,
                       A.STRATEGY[strategy], labels, gat_heads=heads)
        tr.set_params(aptgen.weights(cfg))
        if heads:
            tr.set_attention(np.full(dims[1], 0.1, np.float32), np.full(dims[1], -0.1, np.float32))
        tr.set_epoch(train, 0)
        for s in range(2):
            tr.step(s, update=True)
        ctx.sync()
        print(f"{strategy} C={C} {dtype} heads={heads} dims={dims}: loss {tr.loss():.5f}", flush=True)
        for h in (tr, fs, gr):
            h.close()
        ctx.close()
    L = A.lib()
    print("gemm selftests", [round(L.apt_selftest_gemm(f, am, bm, 200, 70, 100, acc), 9)
                             for f in (0, 1) for am in (0, 1) for bm in (0, 1) for acc in (0, 1)], flush=True)
    print("sort selftest", L.apt_selftest_sort(5000, 3, 4), flush=True)


if __name__ == "__main__":
    main()
