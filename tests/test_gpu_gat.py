"""GPU parity of the GAT first layer under every strategy (-m gpu).

The CUDA path (gat.cu: aggregate-first, online softmax, per-strategy exchanges) is
compared with oracle/gat.py's definition-order fp64 layer on each requester's own
sampled block; the all-reduced gradients with the sum over ranks of the oracle's
per-rank gradients (the strategies are re-partitionings of the same sums).
Tolerances: BASELINE north_star (fp32 rtol 1e-5 / atol 1e-6, bf16 rtol 2e-2) with
the atol floors of DESIGN.md §13.
"""
import numpy as np
import pytest

import aptgen
import oracle
from oracle import gat, model

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

HEADS = 4
TOL = {"f32": dict(rtol=1e-5, atol=1e-5), "bf16": dict(rtol=2e-2, atol=2e-3)}


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
    tol = TOL[dtype]
    dW = db = das = dad = 0.0
    dh_dev = []
    for r in range(C):
        blocks, blk, x, c, emu, (a_s, a_d) = _layer1_oracle(cfg, g, seeds[r], params, att, dims, relu, dtype,
                                                            (part, C) if strategy == "SNP" else None)
        h_cmp = emu["h"]
        got = tr.read("H", 1, rank=r)
        assert got.shape == c["h"].shape
        assert np.allclose(got, h_cmp, **tol), f"rank {r}: max |diff| {np.abs(got - h_cmp).max()}"
        n1, d1 = c["h"].shape
        dh = rng.normal(size=(n1, d1)).astype(np.float32)
        # the ReLU mask as the path's own pre-activation sets it (rounding points included)
        gpre = dh.astype(np.float64) * ((emu["pre"] > 0) if relu else 1.0)
        if dtype == "bf16":
            gpre = oracle.bf16_round(gpre)                     # g is read as its bf16 copy (reading R4)
        gW, ga_s, ga_d, gb_ = gat.backward(blk.indptr, blk.indices, x, blk.n_dst, params[0][0], a_s, a_d, c, gpre,
                                           HEADS)
        dW, db, das, dad = dW + gW, db + gb_, das + ga_s.reshape(-1), dad + ga_d.reshape(-1)
        dh_dev.append(torch.as_tensor(dh).cuda())
    tr.layer_bwd(dh_dev, d1)
    atol = tol["atol"] * 100 if dtype == "bf16" else 1e-4       # unit-scale g: sums of ~1e4 products
    rtol = tol["rtol"] if dtype == "bf16" else 1e-4
    for r in (0, C - 1):
        gdW = tr.read("dW", 1, rank=r)
        assert np.allclose(gdW, dW, rtol=rtol, atol=atol), f"dW max |diff| {np.abs(gdW - dW).max()}"
        assert np.allclose(tr.read("db", 1, rank=r)[0], db, rtol=rtol, atol=atol)
        dA = tr.read("dA", 1, rank=r)[0]
        assert np.allclose(dA[:d1], das, rtol=rtol, atol=atol), f"da_src max |diff| {np.abs(dA[:d1] - das).max()}"
        assert np.allclose(dA[d1:], dad, rtol=rtol, atol=atol), f"da_dst max |diff| {np.abs(dA[d1:] - dad).max()}"


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
    assert abs(got - loss) <= 1e-4 * abs(loss) + 1e-5, (got, loss)
    a0 = tr.get_attention(0)
    W0 = tr.get_params(0)[0][0]
    tr.step(0, update=True)
    a1 = tr.get_attention(0)
    W1 = tr.get_params(0)[0][0]
    assert np.all(np.isfinite(a1[0])) and not np.array_equal(a0[0], a1[0])
    if strategy != "NFP":
        assert not np.array_equal(W0, W1)
