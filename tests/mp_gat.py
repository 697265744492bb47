"""One process per rank on one B200 (CUDA IPC stands in for NVLink): the GAT first
layer (gat.cu) under every strategy through the multi-process path -- peer-mapped
requester buffers (SNP slots, NFP score sums, t, g), device barriers, peer
all-reduce -- against the oracle.  Launched by tests/test_gpu_multiprocess.py under
torchrun; rank 0 prints RESULT."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import aptgen  # noqa: E402
import oracle  # noqa: E402
from oracle import gat  # noqa: E402
from oracle import strategy as S  # noqa: E402
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A  # noqa: E402

HEADS = 4


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dev = int(os.environ.get("APT_TEST_DEVICE", os.environ.get("LOCAL_RANK", 0)))
    dist.init_process_group("gloo")
    torch.cuda.set_device(dev)
    cfg = aptgen.CONFIGS["tiny"]
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    part = aptgen.partition(g.n, world)
    params = aptgen.weights(cfg)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    d1, F = dims[1], dims[1] // HEADS
    rng = np.random.default_rng(11)
    a_s = (rng.normal(size=d1) * 0.5).astype(np.float32)
    a_d = (rng.normal(size=d1) * 0.5).astype(np.float32)
    K = len(cfg.fanouts)
    errors = []
    for strategy in sys.argv[1].split(","):
        ctx = A.Ctx(rank, world, dev)
        ctx.set_exchange(dist)
        gr = ctx.graph_load(g.indptr, g.indices, part)
        fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, A.F32, cfg.dim, None, cfg.feat_seed)
        tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.F32, 0.1, cfg.sample_seed, cfg.feat_seed,
                       A.STRATEGY[strategy], labels, gat_heads=HEADS)
        tr.set_params(params)
        tr.set_attention(a_s, a_d)
        tr.set_epoch(train, 0)
        tr.layer_fwd(0)
        gb = oracle.global_batch(perm, 0, world, cfg.batch)
        seeds = S.assign_seeds(strategy, gb, part, world, cfg.batch)
        dW = db = das = dad = 0.0
        mine = None
        for r in range(world):
            blk = oracle.sample_blocks(g, seeds[r], cfg.fanouts, cfg.sample_seed, 0)[K - 1]
            x = oracle.features(cfg.feat_seed, blk.src, cfg.dim)
            W1, b1 = params[0]
            c = gat.forward(blk.indptr, blk.indices, x, blk.n_dst, W1, a_s.reshape(HEADS, F).astype(np.float64),
                            a_d.reshape(HEADS, F).astype(np.float64), b1, HEADS, relu=K > 1)
            dh = np.random.default_rng(100 + r).normal(size=c["h"].shape).astype(np.float32)
            gpre = dh.astype(np.float64) * ((c["pre"] > 0) if K > 1 else 1.0)
            gW, gs, gd, gbias = gat.backward(blk.indptr, blk.indices, x, blk.n_dst, W1,
                                            a_s.reshape(HEADS, F).astype(np.float64),
                                            a_d.reshape(HEADS, F).astype(np.float64), c, gpre, HEADS)
            dW, db, das, dad = dW + gW, db + gbias, das + gs.reshape(-1), dad + gd.reshape(-1)
            if r == rank:
                mine = (c["h"], dh)
        tag = f"GAT/{strategy}/rank{rank}"
        h1 = tr.read("H", 1, rank=rank)
        if h1.shape != mine[0].shape or not np.allclose(h1, mine[0], rtol=1e-5, atol=1e-5):
            errors.append(f"{tag}: h1 max err {np.abs(h1 - mine[0]).max() if h1.shape == mine[0].shape else 'shape'}")
        tr.layer_bwd([torch.as_tensor(mine[1]).cuda()], d1)
        try:
            ctx.sync()
        except Exception as e:
            errors.append(f"{tag}: {e}")
        tol = dict(rtol=1e-4, atol=1e-4)
        if strategy != "NFP":
            if not np.allclose(tr.read("dW", 1, rank=rank), dW, **tol):
                errors.append(f"{tag}: dW1 max err {np.abs(tr.read('dW', 1, rank=rank) - dW).max():.3g}")
        else:
            lo, hi = S.col_range(rank, world, cfg.dim)
            if not np.allclose(tr.read("dW", 1, rank=rank)[:, lo:hi], dW[:, lo:hi], **tol):
                errors.append(f"{tag}: dW1 slice")
        if not np.allclose(tr.read("db", 1, rank=rank)[0], db, **tol):
            errors.append(f"{tag}: db1")
        dA = tr.read("dA", 1, rank=rank)[0]
        if not (np.allclose(dA[:d1], das, **tol) and np.allclose(dA[d1:], dad, **tol)):
            errors.append(f"{tag}: da max err {max(np.abs(dA[:d1] - das).max(), np.abs(dA[d1:] - dad).max()):.3g}")
        for h in (tr, fs, gr):
            h.close()
        ctx.close()
    allerr = [None] * world
    dist.all_gather_object(allerr, errors)
    if rank == 0:
        flat = [e for x in allerr for e in x]
        print("RESULT", "OK" if not flat else "FAIL " + "; ".join(flat[:20]), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
