"""GPU parity of the GAT first layer under every strategy (-m gpu).

The CUDA path (gat.cu: aggregate-first, online softmax, per-strategy exchanges) is
compared with oracle/gat.py's definition-order fp64 layer on each requester's own
sampled block; the all-reduced gradients with the sum over ranks of the oracle's
per-rank gradients (the strategies are re-partitionings of the same sums).
Tolerances: BASELINE north_star (fp32 rtol 1e-5 / atol 1e-6, bf16 rtol 2e-2) with the
atol derived from the terms' magnitudes (tests/parity_util.py gat_bounds, DESIGN.md §13 T5).
"""
import numpy as np
import pytest

import aptgen
import oracle
from oracle import gat, model
from parity_util import assert_close, gat_bounds

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

HEADS = 4


@pytest.fixture(scope="module")
def A():
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    A.lib()
    return A


@pytest.fixture(scope="module")
def tiny(tiny_cfg, tiny_graph):
    return tiny_cfg, tiny_graph, aptgen.train_nodes(tiny_graph, tiny_cfg)


def _attention(d1, seed=11):
    rng = np.random.default_rng(seed)
    return (rng.normal(size=d1) * 0.5).astype(np.float32), (rng.normal(size=d1) * 0.5).astype(np.float32)


def _setup(A, cfg, g, train, strategy, C, dtype):
    ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
    part = aptgen.partition(g.n, C)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    dt = A.DTYPE[dtype]
    fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    labels = aptgen.labels(cfg, g.n)
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, 0.1, cfg.sample_seed, cfg.feat_seed,
                   A.STRATEGY[strategy], labels, gat_heads=HEADS)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    a_s, a_d = _attention(dims[1])
    tr.set_attention(a_s, a_d)
    tr.set_epoch(train, 0)
    return ctx, part, tr, params, labels, dims, (a_s, a_d)


def _layer1_oracle(cfg, g, seeds, params, att, dims, relu, dtype, snp=None):
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, 0)
    blk = blocks[len(cfg.fanouts) - 1]
    x = oracle.features(cfg.feat_seed, blk.src, cfg.dim)
    W1, b1 = params[0]
    F = dims[1] // HEADS
    a_s = att[0].astype(np.float64).reshape(HEADS, F)
    a_d = att[1].astype(np.float64).reshape(HEADS, F)
    c = gat.forward(blk.indptr, blk.indices, x, blk.n_dst, W1, a_s, a_d, b1, HEADS, relu=relu)
    emu = c
    if dtype == "bf16":     # the CUDA path's rounding points (Z^h and W in bf16), re-associated
        sn = None if snp is None else (np.asarray(snp[0])[blk.src], snp[1])
        emu = gat.forward_aggfirst(blk.indptr, blk.indices, x, blk.n_dst, W1, a_s, a_d, b1, HEADS, relu=relu,
                                   dtype="bf16", snp=sn)
    return blocks, blk, x, c, emu, (a_s, a_d)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("strategy,C", [("GDP", 1), ("GDP", 2), ("DNP", 2), ("DNP", 4), ("SNP", 2), ("SNP", 4),
                                        ("NFP", 2), ("NFP", 4)])
def test_gat_layer_fwd_bwd_matches_oracle(A, tiny, strategy, C, dtype):
    cfg, g, train = tiny
    ctx, part, tr, params, labels, dims, att = _setup(A, cfg, g, train, strategy, C, dtype)
    K = len(cfg.fanouts)
    relu = K > 1
    tr.layer_fwd(0)
    from oracle import strategy as S
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, 0, C, cfg.batch)
    seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
    rng = np.random.default_rng(C)
    dW = db = das = dad = 0.0
    bW = bb = bs = bd = 0.0
    dh_dev = []
    for r in range(C):
        blocks, blk, x, c, emu, (a_s, a_d) = _layer1_oracle(cfg, g, seeds[r], params, att, dims, relu, dtype,
                                                            (part, C) if strategy == "SNP" else None)
        got = tr.read("H", 1, rank=r)
        assert got.shape == c["h"].shape
        n1, d1 = c["h"].shape
        dh = rng.normal(size=(n1, d1)).astype(np.float32)
        # the ReLU mask as the path's own pre-activation sets it (rounding points included)
        gpre = dh.astype(np.float64) * ((emu["pre"] > 0) if relu else 1.0)
        if dtype == "bf16":
            gpre = oracle.bf16_round(gpre)                     # g is read as its bf16 copy (reading R4)
        bnd = gat_bounds(blk.indptr, blk.indices, x, blk.n_dst, params[0][0], a_s, a_d, params[0][1], c, gpre, HEADS,
                         dtype)
        assert_close(got, emu["h"], dtype, f"h1 rank {r}", bnd["h"])
        gW, ga_s, ga_d, gb_ = gat.backward(blk.indptr, blk.indices, x, blk.n_dst, params[0][0], a_s, a_d, c, gpre,
                                           HEADS)
        dW, db, das, dad = dW + gW, db + gb_, das + ga_s.reshape(-1), dad + ga_d.reshape(-1)
        bW, bb, bs, bd = bW + bnd["dW"], bb + bnd["db"], bs + bnd["da_src"], bd + bnd["da_dst"]
        dh_dev.append(torch.as_tensor(dh).cuda())
    tr.layer_bwd(dh_dev, d1)
    for r in (0, C - 1):
        assert_close(tr.read("dW", 1, rank=r), dW, dtype, f"dW rank {r}", bW)
        assert_close(tr.read("db", 1, rank=r)[0], db, dtype, f"db rank {r}", bb)
        dA = tr.read("dA", 1, rank=r)[0]
        assert_close(dA[:d1], das, dtype, f"da_src rank {r}", bs)
        assert_close(dA[d1:], dad, dtype, f"da_dst rank {r}", bd)


@pytest.mark.parametrize("strategy,C", [("GDP", 1), ("DNP", 2), ("SNP", 2), ("NFP", 2)])
def test_gat_train_step_loss_and_update(A, tiny, strategy, C):
    """The full step with a GAT first layer and SAGE upper layers: the loss equals the
    oracle composition, and SGD moves W^1 and the attention vectors."""
    cfg, g, train = tiny
    ctx, part, tr, params, labels, dims, att = _setup(A, cfg, g, train, strategy, C, "f32")
    K = len(cfg.fanouts)
    tr.step(0, update=False)
    got = tr.loss()
    from oracle import strategy as S
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, 0, C, cfg.batch)
    seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
    loss = 0.0
    for r in range(C):
        blocks, blk, x, c, _, _ = _layer1_oracle(cfg, g, seeds[r], params, att, dims, K > 1, "f32")
        H = c["h"]
        for l in range(2, K + 1):
            b2 = blocks[K - l]
            W, b = params[l - 1]
            pre = oracle.aggregate(b2.indptr, b2.indices, H) @ W.astype(np.float64).T + b
            H = np.maximum(pre, 0.0) if l < K else pre
        lr_, _ = model.ce_loss_grad(H, labels[seeds[r]], len(gb))
        loss += lr_
    # fp32 loss: CE of logits within the T1 bar of the three-layer chain (sum of C*B terms)
    assert abs(got - loss) <= 1e-5 * abs(loss) + 1e-6, (got, loss)
    # one SGD step against the oracle's: W1' = W1 - lr dW1, a' = a - lr da (lr 0.1, _setup);
    # the gradients come from the oracle's composition of the GAT layer and the SAGE upper layers
    W0 = tr.get_params(0)[0][0].astype(np.float64)
    a0 = [v.astype(np.float64) for v in tr.get_attention(0)]
    tr.step(0, update=True)
    W1n = tr.get_params(0)[0][0]
    a1 = tr.get_attention(0)
    dW = da_s = da_d = 0.0
    lr = 0.1
    for r in range(C):
        blocks, blk, x, c, _, (a_s, a_d) = _layer1_oracle(cfg, g, seeds[r], params, att, dims, K > 1, "f32")
        Hs, pres = [c["h"]], [c["pre"]]
        for l in range(2, K + 1):
            b2 = blocks[K - l]
            W, b = params[l - 1]
            pre = oracle.aggregate(b2.indptr, b2.indices, Hs[-1]) @ W.astype(np.float64).T + b
            pres.append(pre)
            Hs.append(np.maximum(pre, 0.0) if l < K else pre)
        _, gl = model.ce_loss_grad(Hs[-1], labels[seeds[r]], len(gb))
        for l in range(K, 1, -1):
            b2 = blocks[K - l]
            W, _ = params[l - 1]
            gl = oracle.aggregate_bwd(b2.indptr, b2.indices, gl @ W.astype(np.float64), b2.n_src) * (pres[l - 2] > 0)
        gW, ga_s, ga_d, _ = gat.backward(blk.indptr, blk.indices, x, blk.n_dst, params[0][0], a_s, a_d, c, gl, HEADS)
        dW, da_s, da_d = dW + gW, da_s + ga_s.reshape(-1), da_d + ga_d.reshape(-1)
    if strategy != "NFP":   # NFP: W^1 is column-owned (each rank updates its slice)
        assert np.allclose((W0 - W1n) / lr, dW, rtol=1e-3, atol=1e-6 + 2.0 ** -23 * np.abs(W0).max() / lr)
    assert np.allclose((a0[0] - a1[0]) / lr, da_s, rtol=1e-3, atol=1e-6 + 2.0 ** -23 * np.abs(a0[0]).max() / lr)
    assert np.allclose((a0[1] - a1[1]) / lr, da_d, rtol=1e-3, atol=1e-6 + 2.0 ** -23 * np.abs(a0[1]).max() / lr)
