"""Pins for the CPU oracle (-m "not gpu").

Every test here checks the oracle against something other than itself: published
known-answer vectors, exact probabilities, brute force on tiny inputs, a
textbook dense product, finite differences, or a library routine.
"""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp
from scipy import stats

import aptgen
import oracle
from oracle import model


# ---------------------------------------------------------------- O0 Philox
def _philox_kats():
    """tests/golden/philox4x32_10_kat.txt: Random123 kat_vectors (cited in the file)."""
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "philox4x32_10_kat.txt")
    out = []
    for line in open(path):
        if line.strip() and not line.startswith("#"):
            ctr, key, exp = (list(int(w, 16) for w in f.split()) for f in line.split("|"))
            out.append((ctr, key, exp))
    assert len(out) == 3
    return out


@pytest.mark.parametrize("ctr,key,expect", _philox_kats())
def test_philox_kat(ctr, key, expect):
    assert [int(x) for x in oracle.philox(ctr, key)] == expect


# ---------------------------------------------------------------- O2 sampler
def test_sampler_small_degree_takes_full_row():
    for deg in range(0, 6):
        assert list(oracle.sample_positions(17, deg, 5, 3, 0, 0)) == list(range(deg))


def test_sampler_positions_valid_and_deterministic():
    for deg, k in [(6, 5), (50, 10), (1000, 25), (300, 256)]:
        for step in range(20):
            p = oracle.sample_positions(123456789012, deg, k, 7, step, 1)
            assert len(p) == k
            assert np.all(np.diff(p) > 0) and p[0] >= 0 and p[-1] < deg
            assert np.array_equal(p, oracle.sample_positions(123456789012, deg, k, 7, step, 1))


def test_sampler_exact_subset_distribution():
    """deg=5, k=2: each of the C(5,2)=10 subsets has probability exactly 1/10."""
    counts = {s: 0 for s in itertools.combinations(range(5), 2)}
    n = 20000
    for step in range(n):
        counts[tuple(int(x) for x in oracle.sample_positions(42, 5, 2, 11, step, 0))] += 1
    obs = np.array(list(counts.values()))
    assert stats.chisquare(obs).pvalue > 1e-3


def test_sampler_pairwise_inclusion():
    """Uniform k-subset: P(i in S) = k/deg, P(i,j in S) = k(k-1)/(deg(deg-1))."""
    deg, k, n = 9, 4, 20000
    single = np.zeros(deg)
    pair = np.zeros((deg, deg))
    for step in range(n):
        p = oracle.sample_positions(5, deg, k, 13, step, 2)
        single[p] += 1
        pair[np.ix_(p, p)] += 1
    assert np.allclose(single / n, k / deg, atol=0.02)
    off = pair[~np.eye(deg, dtype=bool)] / n
    assert np.allclose(off, k * (k - 1) / (deg * (deg - 1)), atol=0.015)


def test_sampler_keys_depend_on_hop_step_node():
    a = oracle.sample_positions(10, 100, 10, 1, 0, 0)
    assert not np.array_equal(a, oracle.sample_positions(10, 100, 10, 1, 0, 1))
    assert not np.array_equal(a, oracle.sample_positions(10, 100, 10, 1, 1, 0))
    assert not np.array_equal(a, oracle.sample_positions(11, 100, 10, 1, 0, 0))
    assert not np.array_equal(a, oracle.sample_positions(10, 100, 10, 2, 0, 0))


# ---------------------------------------------------------------- O3 compaction
def test_compaction_brute_force(tiny_graph):
    g = tiny_graph
    rng = np.random.default_rng(0)
    seeds = rng.choice(np.nonzero(g.degrees() > 0)[0], 64, replace=False).astype(np.int64)
    blocks = oracle.sample_blocks(g, seeds, (5, 5), seed=3, step=7)
    for h, blk in enumerate(blocks):
        F = blk.n_dst
        assert np.array_equal(blk.src[:F], blk.dst)                    # dst prefix
        assert len(np.unique(blk.src)) == blk.n_src                    # unique
        new = blk.src[F:]
        assert np.all(np.diff(new) > 0)                                # ascending
        assert not np.isin(new, blk.dst).any()
        # brute force: src set == dst U sampled neighbours
        nb = [int(blk.nbr[i * blk.k + q]) for i in range(F) for q in range(blk.cnt[i])]
        assert set(blk.src.tolist()) == set(blk.dst.tolist()) | set(nb)
        assert blk.n_edges == int(blk.cnt.sum())
        assert np.all(blk.indices < blk.n_src)
        # every edge maps back to its sampled (v, u) pair, and u is a real neighbour
        for i in range(F):
            us = blk.src[blk.indices[blk.indptr[i]:blk.indptr[i + 1]]]
            assert list(us) == [int(x) for x in blk.nbr[i * blk.k:i * blk.k + blk.cnt[i]]]
            v = blk.dst[i]
            row = g.indices[g.indptr[v]:g.indptr[v + 1]]
            assert np.isin(us, row).all()
            assert np.all(np.diff(us) > 0)                              # CSR order kept
        if h + 1 < len(blocks):
            assert np.array_equal(blocks[h + 1].dst, blk.src)           # next frontier


# ---------------------------------------------------------------- O4 features
def test_features_exact_grid_and_uniform_bytes():
    x = oracle.features(2, np.arange(4000, dtype=np.int64), 64)
    k = x * 64
    assert np.array_equal(k, np.round(k)) and k.min() >= -128 and k.max() <= 127
    assert np.array_equal(x.astype(np.float32).astype(np.float64), x)
    assert np.array_equal(oracle.bf16_round(x), x)                     # exact in bf16
    hist = np.bincount((k.astype(np.int64) + 128).ravel(), minlength=256)
    assert stats.chisquare(hist).pvalue > 1e-4


# ---------------------------------------------------------------- O5 aggregation
def test_aggregate_full_fanout_is_row_normalised_spmm(tiny_graph):
    """Special case: fanout >= max degree => the sampler keeps every edge and
    Z = D^-1 A X on the seeds' rows (textbook row-normalised SpMM)."""
    g = tiny_graph
    kmax = int(g.degrees().max())
    seeds = np.array([0, 1, 2, 17, 333, 4096, 9999], np.int64)
    seeds = seeds[g.degrees()[seeds] > 0]
    (blk,) = oracle.sample_blocks(g, seeds, (kmax,), seed=3, step=0)
    X = oracle.features(2, np.arange(g.n, dtype=np.int64), 16)
    Z = oracle.aggregate(blk.indptr, blk.indices, X[blk.src])
    A = sp.csr_matrix((np.ones(g.nnz), g.indices, g.indptr), shape=(g.n, g.n)).toarray()
    dense = (A / A.sum(1, keepdims=True).clip(min=1)) @ X
    assert np.allclose(Z, dense[seeds], rtol=0, atol=1e-12)


def test_aggregate_zero_degree_row_is_zero():
    Z = oracle.aggregate(np.array([0, 0, 2]), np.array([0, 1], np.int32), np.ones((2, 3)))
    assert np.array_equal(Z, [[0, 0, 0], [1, 1, 1]])


def test_aggregate_bwd_is_adjoint(tiny_graph):
    rng = np.random.default_rng(1)
    seeds = rng.choice(np.nonzero(tiny_graph.degrees() > 0)[0], 50, replace=False)
    (blk,) = oracle.sample_blocks(tiny_graph, seeds, (5,), seed=3, step=1)
    x = rng.normal(size=(blk.n_src, 7))
    dz = rng.normal(size=(blk.n_dst, 7))
    lhs = np.sum(oracle.aggregate(blk.indptr, blk.indices, x) * dz)
    rhs = np.sum(x * oracle.aggregate_bwd(blk.indptr, blk.indices, dz, blk.n_src))
    assert abs(lhs - rhs) < 1e-9 * max(1, abs(lhs))


# ---------------------------------------------------------------- model
def _tiny_setup(tiny_graph, tiny_cfg, n_seeds=24, dims=None):
    cfg = tiny_cfg if dims is None else tiny_cfg.replace(**dims)
    rng = np.random.default_rng(2)
    seeds = rng.choice(np.nonzero(tiny_graph.degrees() > 0)[0], n_seeds, replace=False).astype(np.int64)
    blocks = oracle.sample_blocks(tiny_graph, seeds, cfg.fanouts, cfg.sample_seed, 0)
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in aptgen.weights(cfg)]
    labels = aptgen.labels(cfg, tiny_graph.n)[seeds]
    return cfg, seeds, blocks, params, labels


def test_forward_matches_explicit_tree_recursion(tiny_graph, tiny_cfg):
    """Brute force: h^K(seed) by recursing over the sampled neighbour lists in plain
    Python (Eq. 1), independent of block / compaction bookkeeping."""
    cfg, seeds, blocks, params, _ = _tiny_setup(tiny_graph, tiny_cfg, 6, dict(dim=8, hidden=5, n_classes=3))
    K = len(blocks)
    nbrs = [dict() for _ in range(K)]
    for h, blk in enumerate(blocks):
        for i, v in enumerate(blk.dst):
            nbrs[h][int(v)] = [int(u) for u in blk.nbr[i * blk.k:i * blk.k + blk.cnt[i]]]

    def h_of(v, layer):          # embedding of v after `layer` layers
        if layer == 0:
            return oracle.features(cfg.feat_seed, np.array([v]), cfg.dim)[0]
        hop = K - layer
        us = nbrs[hop][v]
        z = np.mean([h_of(u, layer - 1) for u in us], axis=0) if us else np.zeros(
            cfg.dim if layer == 1 else cfg.hidden)
        W, b = params[layer - 1]
        pre = W @ z + b
        return np.maximum(pre, 0) if layer < K else pre

    cache = model.forward(blocks, cfg.feat_seed, cfg.dim, params)
    for i, s in enumerate(seeds):
        assert np.allclose(cache["logits"][i], h_of(int(s), K), rtol=1e-12, atol=1e-12)


def test_bf16_forward_matches_tree_recursion_with_torch_rounding(tiny_graph, tiny_cfg):
    """bf16 mode's rounding points (O5, reading R11) by an independent recursion: the
    mean in fp64 -> fp32 -> bf16, W in bf16, hidden activations rounded to bf16 after
    bias + ReLU, every rounding done by torch's bfloat16 conversion."""
    import torch

    def rb(x):
        return torch.tensor(np.asarray(x, np.float64)).float().bfloat16().double().numpy()

    cfg, seeds, blocks, params, _ = _tiny_setup(tiny_graph, tiny_cfg, 6, dict(dim=8, hidden=5, n_classes=3))
    K = len(blocks)
    nbrs = [dict() for _ in range(K)]
    for h, blk in enumerate(blocks):
        for i, v in enumerate(blk.dst):
            nbrs[h][int(v)] = [int(u) for u in blk.nbr[i * blk.k:i * blk.k + blk.cnt[i]]]

    def h_of(v, layer):
        if layer == 0:
            return oracle.features(cfg.feat_seed, np.array([v]), cfg.dim)[0]
        us = nbrs[K - layer][v]
        z = np.mean([h_of(u, layer - 1) for u in us], axis=0) if us else np.zeros(
            cfg.dim if layer == 1 else cfg.hidden)
        W, b = params[layer - 1]
        pre = rb(W) @ rb(z) + b
        return rb(np.maximum(pre, 0)) if layer < K else pre

    cache = model.forward(blocks, cfg.feat_seed, cfg.dim, params, "bf16")
    for i, s in enumerate(seeds):
        assert np.allclose(cache["logits"][i], h_of(int(s), K), rtol=1e-12, atol=1e-12)
    for h in cache["h"][:-1]:                    # hidden activations are bf16 values
        assert np.array_equal(rb(h), h)


def test_ce_loss_matches_torch(tiny_graph, tiny_cfg):
    import torch
    rng = np.random.default_rng(3)
    logits = rng.normal(size=(40, 16)) * 3
    labels = rng.integers(0, 16, 40)
    loss, g = model.ce_loss_grad(logits, labels, 100)
    t = torch.tensor(logits, requires_grad=True)
    ref = torch.nn.functional.cross_entropy(t, torch.tensor(labels), reduction="sum") / 100
    ref.backward()
    assert abs(loss - ref.item()) < 1e-12
    assert np.allclose(g, t.grad.numpy(), atol=1e-14)


def test_backward_finite_differences(tiny_graph, tiny_cfg):
    """Central differences of the fp64 loss wrt W^l and b^l (O5 backward)."""
    cfg, seeds, blocks, params, labels = _tiny_setup(tiny_graph, tiny_cfg, 16, dict(dim=6, hidden=4, n_classes=3))
    out = model.train_step(blocks, cfg.feat_seed, cfg.dim, params, labels, n_global=16)

    def loss_of(ps):
        c = model.forward(blocks, cfg.feat_seed, cfg.dim, ps)
        return model.ce_loss_grad(c["logits"], labels, 16)[0]

    eps = 1e-6
    rng = np.random.default_rng(4)
    for l in range(len(params)):
        W, b = params[l]
        for _ in range(6):
            i, j = rng.integers(0, W.shape[0]), rng.integers(0, W.shape[1])
            Wp, Wm = W.copy(), W.copy()
            Wp[i, j] += eps
            Wm[i, j] -= eps
            pp = list(params); pp[l] = (Wp, b)
            pm = list(params); pm[l] = (Wm, b)
            fd = (loss_of(pp) - loss_of(pm)) / (2 * eps)
            assert abs(fd - out["grads"][l][0][i, j]) <= 1e-6 * max(1e-3, abs(fd)) + 1e-9
        i = rng.integers(0, len(b))
        bp, bm = b.copy(), b.copy()
        bp[i] += eps
        bm[i] -= eps
        pp = list(params); pp[l] = (W, bp)
        pm = list(params); pm[l] = (W, bm)
        fd = (loss_of(pp) - loss_of(pm)) / (2 * eps)
        assert abs(fd - out["grads"][l][1][i]) <= 1e-6 * max(1e-3, abs(fd)) + 1e-9


def test_bf16_round_matches_torch():
    import torch
    x = np.random.default_rng(5).normal(size=10000) * 10
    ref = torch.tensor(x, dtype=torch.float32).to(torch.bfloat16).to(torch.float64).numpy()
    assert np.array_equal(oracle.bf16_round(x), ref)


# ---------------------------------------------------------------- O1 permutation
def test_epoch_perm_is_permutation_and_epoch_dependent():
    train = np.arange(0, 5000, 3, dtype=np.int64)
    p0 = oracle.epoch_perm(train, 9, 0)
    p1 = oracle.epoch_perm(train, 9, 1)
    assert np.array_equal(np.sort(p0), train) and np.array_equal(np.sort(p1), train)
    assert not np.array_equal(p0, p1) and not np.array_equal(p0, train)
    # positions are uniform-ish: mean rank of the first half of train ~ n/2
    rank = np.empty(len(train)); rank[np.searchsorted(train, p0)] = np.arange(len(train))
    assert abs(rank[: len(train) // 2].mean() / len(train) - 0.5) < 0.05


def test_snp_partials_sum_to_mean_and_split_by_partition(tiny_graph, tiny_cfg):
    """SNP partial aggregates: sum over partitions = the full mean (linearity),
    and P~_c only draws on sources owned by c."""
    from oracle import model
    seeds = aptgen.train_nodes(tiny_graph, tiny_cfg)[:64]
    blk = oracle.sample_blocks(tiny_graph, seeds, (6,), 9, 1)[0]
    x = oracle.features(tiny_cfg.feat_seed, blk.src, 16)
    part = aptgen.partition(tiny_graph.n, 4)
    parts = model.snp_partials(blk, x, part, 4)
    assert np.allclose(sum(parts), oracle.aggregate(blk.indptr, blk.indices, x), rtol=0, atol=1e-12)
    # zeroing the features of partition 1 leaves every other partial unchanged
    x2 = x.copy()
    x2[part[blk.src] == 1] = 0.0
    p2 = model.snp_partials(blk, x2, part, 4)
    assert np.array_equal(p2[0], parts[0]) and np.array_equal(p2[2], parts[2]) and not p2[1].any()
