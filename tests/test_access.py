"""Node access frequencies (Table 3; reading R12) and the excess
cache's hot list: oracle pins (-m "not gpu"), the host-side apt_hot_rows (no GPU
needed) and GPU parity of apt_access_counts (bit-exact)."""
import numpy as np
import pytest
import scipy.sparse as sp

import aptgen
from oracle import strategy as S


def _adj(g):
    return sp.csr_matrix((np.ones(len(g.indices)), g.indices, g.indptr), shape=(g.n, g.n))


def test_access_counts_full_fanout_is_two_hop_neighbourhood(tiny_graph, tiny_cfg):
    """With fanouts above the maximum degree the sampler takes every neighbour (O2), so
    the layer-1 sources of a rank are N(seeds ∪ N(seeds)) -- computed here straight from
    the CSR with scipy, per (step, rank)."""
    g = tiny_graph
    train = aptgen.train_nodes(g, tiny_cfg)
    kmax = int(np.diff(g.indptr).max()) + 1
    C, B, steps = 2, 64, 3
    got = S.access_counts(g, train, (kmax, kmax), tiny_cfg.sample_seed, 0, C, B, steps)
    import oracle
    perm = oracle.epoch_perm(train, tiny_cfg.sample_seed, 0)
    A = _adj(g)
    want = np.zeros(g.n, np.int64)
    for t in range(steps):
        gb = perm[t * C * B:(t + 1) * C * B]
        for r in range(C):
            s = np.zeros(g.n)
            s[gb[r * B:(r + 1) * B]] = 1
            f1 = (s + A @ s) > 0                  # hop-1 frontier: seeds and their neighbours
            want += (A @ f1.astype(float)) > 0    # layer-1 sources: neighbours of the frontier
    assert np.array_equal(got, want)


def test_skew_table_closed_form():
    # 100 nodes: node i accessed 100 - i times -> bucket shares are exact sums
    c = np.arange(100, 0, -1)
    tab = S.skew_table(c)
    tot = c.sum()
    assert np.allclose(tab, [c[:1].sum() / tot, c[1:5].sum() / tot, c[5:10].sum() / tot,
                             c[10:20].sum() / tot, c[20:50].sum() / tot, c[50:].sum() / tot])
    assert abs(sum(tab) - 1) < 1e-12
    assert S.skew_table(np.ones(1000))[0] == pytest.approx(0.01)   # uniform access: no skew


def test_hot_rows_matches_lexsort():
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    rng = np.random.default_rng(0)
    c = rng.integers(0, 6, 5000).astype(np.int32)
    want = np.lexsort((np.arange(len(c)), -c.astype(np.int64)))[:700]
    assert np.array_equal(A.hot_rows(c, 700), want)


@pytest.mark.gpu
@pytest.mark.parametrize("C", [1, 2])
def test_access_counts_bit_exact(tiny_graph, tiny_cfg, C):
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    g, cfg = tiny_graph, tiny_cfg
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    ctx = A.Ctx(0 if C == 1 else -1, C, 0)
    part = np.minimum(np.arange(g.n) * C // g.n, C - 1).astype(np.int32)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    fs = ctx.fstore_create(gr, A.GDP, A.BF16, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.BF16, 0.1, cfg.sample_seed, cfg.feat_seed,
                   A.GDP, labels)
    tr.set_epoch(train, 0)
    got = tr.access_counts(4)
    want = S.access_counts(g, train, cfg.fanouts, cfg.sample_seed, 0, C, cfg.batch, 4)
    assert np.array_equal(got, want)
    assert got.sum() > 0
