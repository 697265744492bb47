"""Pins for the GAT oracle (oracle/gat.py, readings G1-G4), -m "not gpu".

Each test checks the oracle against something other than itself: a closed form
worked by hand, the mean aggregation of the C oracle (alpha uniform when the
attention vectors are zero), scipy's softmax, central finite differences of the
loss, and invariances (neighbour order, re-association).
"""
import numpy as np
import pytest
from scipy.special import softmax

import aptgen
import oracle
from oracle import gat


def _rand_block(rng, n_dst=7, n_new=9, max_deg=5):
    n_src = n_dst + n_new
    deg = rng.integers(0, max_deg + 1, n_dst)
    deg[0] = 0                                          # G3: an empty row
    deg[1] = 1                                          # a single neighbour
    indptr = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    indices = np.concatenate([rng.choice(n_src, size=k, replace=False) for k in deg]).astype(np.int32)
    return indptr, indices, n_src


def _params(rng, d, H, F, scale=0.5):
    W = rng.normal(size=(H * F, d)) * scale
    a_s = rng.normal(size=(H, F))
    a_d = rng.normal(size=(H, F))
    b = rng.normal(size=H * F) * 0.1
    return W, a_s, a_d, b


def test_closed_form_two_neighbours():
    # one dst (node 0) with neighbours 1, 2; d = 1, one head, F = 1, W = [[2]]:
    # Y = 2x; e_u = LeakyReLU(a_s*Y_u + a_d*Y_0); alpha = softmax(e); pre = sum alpha Y + b
    x = np.array([[1.0], [0.5], [-1.5]])
    W, a_s, a_d, b = np.array([[2.0]]), np.array([[1.0]]), np.array([[0.25]]), np.array([0.125])
    c = gat.forward(np.array([0, 2]), np.array([1, 2]), x, 1, W, a_s, a_d, b, heads=1, relu=False)
    s1 = 1.0 * 1.0 + 0.25 * 2.0          # 1.5 (> 0)
    s2 = 1.0 * -3.0 + 0.25 * 2.0         # -2.5 -> LeakyReLU -0.5
    e1, e2 = s1, 0.2 * s2
    a1 = np.exp(e1) / (np.exp(e1) + np.exp(e2))
    expect = a1 * 1.0 + (1 - a1) * -3.0 + 0.125
    assert c["pre"][0, 0] == pytest.approx(expect, rel=1e-14)


def test_zero_attention_is_the_mean_aggregation():
    # a_src = a_dst = 0 => every score is 0 => alpha uniform => pre = W mean(x) + b,
    # with the mean taken by the C oracle's aggregation (O5)
    rng = np.random.default_rng(1)
    indptr, indices, n_src = _rand_block(rng)
    d, H, F = 6, 2, 3
    x = rng.normal(size=(n_src, d))
    W, _, _, b = _params(rng, d, H, F)
    z = np.zeros((H, F))
    c = gat.forward(indptr, indices, x, len(indptr) - 1, W, z, z, b, H, relu=False)
    mean = oracle.aggregate(indptr, indices, x)
    assert np.allclose(c["pre"], mean @ W.T + b, rtol=1e-13, atol=1e-13)


def test_softmax_rows_match_scipy_and_single_neighbour_is_one():
    rng = np.random.default_rng(2)
    indptr, indices, n_src = _rand_block(rng)
    e = rng.normal(size=(len(indices), 3)) * 4
    al = gat.edge_softmax(indptr, e)
    for v in range(len(indptr) - 1):
        a, b = indptr[v], indptr[v + 1]
        if b > a:
            assert np.allclose(al[a:b], softmax(e[a:b], axis=0), rtol=1e-14, atol=0)
    assert np.all(al[indptr[1]:indptr[2]] == 1.0)


def test_neighbour_order_invariance():
    rng = np.random.default_rng(3)
    indptr, indices, n_src = _rand_block(rng)
    d, H, F = 5, 4, 2
    x = rng.normal(size=(n_src, d))
    P = _params(rng, d, H, F)
    base = gat.forward(indptr, indices, x, len(indptr) - 1, *P, H)
    perm_idx = indices.copy()
    for v in range(len(indptr) - 1):
        perm_idx[indptr[v]:indptr[v + 1]] = rng.permutation(indices[indptr[v]:indptr[v + 1]])
    other = gat.forward(indptr, perm_idx, x, len(indptr) - 1, *P, H)
    assert np.allclose(base["pre"], other["pre"], rtol=1e-13, atol=1e-13)


def test_aggregate_first_equals_definition():
    rng = np.random.default_rng(4)
    indptr, indices, n_src = _rand_block(rng, 11, 20, 6)
    d, H, F = 8, 4, 3
    x = rng.normal(size=(n_src, d))
    P = _params(rng, d, H, F)
    a = gat.forward(indptr, indices, x, len(indptr) - 1, *P, H)
    b = gat.forward_aggfirst(indptr, indices, x, len(indptr) - 1, *P, H)
    assert np.allclose(a["pre"], b["pre"], rtol=1e-12, atol=1e-12)
    assert np.allclose(a["alpha"], b["alpha"], rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("H,F", [(1, 4), (4, 2)])
def test_backward_matches_finite_differences(H, F):
    rng = np.random.default_rng(5 + H)
    indptr, indices, n_src = _rand_block(rng, 6, 8, 4)
    n_dst, d = len(indptr) - 1, 5
    x = rng.normal(size=(n_src, d))
    W, a_s, a_d, b = _params(rng, d, H, F)
    G = rng.normal(size=(n_dst, H * F))

    def loss(W, a_s, a_d, b):       # L = sum G * pre  =>  dL/dpre = G
        return float((G * gat.forward(indptr, indices, x, n_dst, W, a_s, a_d, b, H, relu=False)["pre"]).sum())

    c = gat.forward(indptr, indices, x, n_dst, W, a_s, a_d, b, H, relu=False)
    dW, das, dad, db = gat.backward(indptr, indices, x, n_dst, W, a_s, a_d, c, G, H)
    eps = 1e-6
    for name, P, grad in (("W", W, dW), ("a_src", a_s, das), ("a_dst", a_d, dad), ("b", b, db)):
        num = np.zeros_like(P)
        for i in np.ndindex(P.shape):
            args = {"W": W, "a_s": a_s, "a_d": a_d, "b": b}
            key = {"W": "W", "a_src": "a_s", "a_dst": "a_d", "b": "b"}[name]
            Pp, Pm = P.copy(), P.copy()
            Pp[i] += eps
            Pm[i] -= eps
            args[key] = Pp
            lp = loss(**args)
            args[key] = Pm
            lm = loss(**args)
            num[i] = (lp - lm) / (2 * eps)
        assert np.allclose(grad, num, rtol=1e-6, atol=1e-8), name


def test_bf16_emulation_rounds_only_z_and_w():
    # O4 features are exact in bf16; with W already bf16-representable and Z rounded,
    # the bf16 emulation differs from f32 by at most the bf16 rounding of Z (2^-9 rel)
    rng = np.random.default_rng(6)
    cfg = aptgen.CONFIGS["tiny"]
    indptr, indices, n_src = _rand_block(rng, 9, 12, 5)
    x = oracle.features(cfg.feat_seed, np.arange(n_src), 16)
    W, a_s, a_d, b = _params(rng, 16, 4, 2)
    W = oracle.bf16_round(W)
    f = gat.forward_aggfirst(indptr, indices, x, len(indptr) - 1, W, a_s, a_d, b, 4, dtype="f32")
    h = gat.forward_aggfirst(indptr, indices, x, len(indptr) - 1, W, a_s, a_d, b, 4, dtype="bf16")
    assert np.allclose(oracle.bf16_round(f["Z"]), h["Z"], rtol=0, atol=0)
    bound = np.abs(f["Z"]).reshape(len(f["Z"]), -1).sum(1).max() * np.abs(W).max() * 2.0 ** -8
    assert np.abs(f["pre"] - h["pre"]).max() <= bound


@pytest.mark.parametrize("C", [2, 3])
def test_snp_partial_merge_equals_definition(C):
    # SNP's per-partition softmax state + merge (reading G5) re-associates the same sums
    rng = np.random.default_rng(10 + C)
    indptr, indices, n_src = _rand_block(rng, 12, 20, 6)
    d, H, F = 6, 4, 2
    x = rng.normal(size=(n_src, d))
    P = _params(rng, d, H, F)
    part = rng.integers(0, C, n_src)
    a = gat.forward(indptr, indices, x, len(indptr) - 1, *P, H)
    b = gat.forward_aggfirst(indptr, indices, x, len(indptr) - 1, *P, H, snp=(part, C))
    assert np.allclose(a["pre"], b["pre"], rtol=1e-12, atol=1e-12)
