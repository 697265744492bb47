"""fp64 GAT first layer -- ORACLE (test infrastructure only).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference legs
may import this module.  It shares no code with the CUDA path.

The paper trains GAT [45] next to GraphSAGE ("GAT uses attention for
neighbor aggregation", "a hidden embedding dimension of 8 and 4 attention
heads") and discusses what attention costs each strategy (P:173, 175, 178,
P:225 SegmentedSDDMM, Fig. 10 / P:344).  It does not restate GAT's equations;
this module writes out GAT's layer [45] in its own order, with the readings of
DESIGN.md §3 (G1-G6):

  G1  Y_u = W x_u, W is d' x d, d' = H*F, head h owns rows [hF, (h+1)F);
      e_vu^h = LeakyReLU_0.2(a_src^h . Y_u^h + a_dst^h . Y_v^h) for u in the
      sampled N(v) (no self loop: Eq. 1's N(v), reading Z8);
      alpha_vu^h = softmax over the sampled u of e_vu^h;
      pre_v = concat_h (sum_u alpha_vu^h Y_u^h) + b.
  G2  bias once after the aggregation, ReLU on hidden layers (Z9, Z10).
  G3  a destination with no sampled neighbour gets pre_v = b.
  G4  heads are concatenated; no attention dropout, no residual.
  G5  SNP partial attention: per source partition, the softmax
      state (max, sum) and the normalised partial sum travel with the partial
      projection; the requester merges them (online-softmax combine).

``forward`` / ``backward`` follow the definition step by step (project, score,
softmax, weighted sum; then the chain rule in reverse).  ``forward_aggfirst``
re-associates the same sums the way the CUDA path does (per-head weighted sums of
x, then the projection) so that the bf16 mode's rounding points -- Z^h -> bf16,
W -> bf16 -- can be emulated; without rounding it equals ``forward`` (tested).
"""
from __future__ import annotations

import numpy as np

from . import bf16_round

SLOPE = 0.2      # LeakyReLU negative slope of GAT [45]


def _rows(indptr):
    deg = np.diff(indptr)
    return np.repeat(np.arange(len(deg)), deg), deg


def _leaky(s):
    return np.where(s > 0, s, SLOPE * s)


def edge_softmax(indptr, e):
    """alpha[i] = exp(e[i]) / sum over the edges of i's destination row of exp(e),
    per head (columns of e).  Max-subtracted, written as a loop over rows."""
    alpha = np.zeros_like(e)
    for v in range(len(indptr) - 1):
        a, b = indptr[v], indptr[v + 1]
        if b > a:
            x = e[a:b] - e[a:b].max(axis=0, keepdims=True)
            ex = np.exp(x)
            alpha[a:b] = ex / ex.sum(axis=0, keepdims=True)
    return alpha


def forward(indptr, indices, x_src, n_dst, W, a_src, a_dst, b, heads, relu=True):
    """G1-G4 in the definition order.  x_src [n_src x d] (dst rows are the prefix),
    W [d' x d], a_src / a_dst [H x F], b [d'].  Returns a cache dict with Y, el, er,
    s (pre-LeakyReLU score), alpha (per edge, per head), pre, h."""
    W = np.asarray(W, np.float64)
    H = heads
    dp = W.shape[0]
    F = dp // H
    x = np.asarray(x_src, np.float64)
    Y = x @ W.T                                             # project every source row
    Yh = Y.reshape(len(x), H, F)
    el = np.einsum("uhf,hf->uh", Yh, np.asarray(a_src, np.float64))
    er = np.einsum("uhf,hf->uh", Yh[:n_dst], np.asarray(a_dst, np.float64))
    rows, _ = _rows(indptr)
    s = el[indices] + er[rows]                               # [E x H]
    alpha = edge_softmax(indptr, _leaky(s))
    agg = np.zeros((n_dst, H, F))
    np.add.at(agg, rows, alpha[:, :, None] * Yh[indices])
    pre = agg.reshape(n_dst, dp) + np.asarray(b, np.float64)
    h = np.maximum(pre, 0.0) if relu else pre
    return {"Y": Y, "el": el, "er": er, "s": s, "alpha": alpha, "pre": pre, "h": h, "rows": rows}


def backward(indptr, indices, x_src, n_dst, W, a_src, a_dst, cache, g, heads):
    """Chain rule of ``forward`` given g = dL/dpre [n_dst x d'].  Returns
    (dW, da_src, da_dst, db).  Layer 1 has no dX (features are constant)."""
    W = np.asarray(W, np.float64)
    H = heads
    dp = W.shape[0]
    F = dp // H
    x = np.asarray(x_src, np.float64)
    Yh = cache["Y"].reshape(len(x), H, F)
    alpha, s, rows = cache["alpha"], cache["s"], cache["rows"]
    gh = np.asarray(g, np.float64).reshape(n_dst, H, F)
    # pre_v^h = sum_u alpha_vu^h Y_u^h
    dalpha = np.einsum("ehf,ehf->eh", gh[rows], Yh[indices])
    t = np.zeros((n_dst, H))
    np.add.at(t, rows, alpha * dalpha)
    de = alpha * (dalpha - t[rows])                          # softmax backward
    ds = de * np.where(s > 0, 1.0, SLOPE)                    # LeakyReLU backward
    dY = np.zeros_like(Yh)
    np.add.at(dY, indices, alpha[:, :, None] * gh[rows])     # through the weighted sum
    del_ = np.zeros((len(x), H))
    np.add.at(del_, indices, ds)                             # d el_u
    der = np.zeros((n_dst, H))
    np.add.at(der, rows, ds)                                 # d er_v
    a_src = np.asarray(a_src, np.float64)
    a_dst = np.asarray(a_dst, np.float64)
    dY += del_[:, :, None] * a_src[None]
    dY[:n_dst] += der[:, :, None] * a_dst[None]
    da_src = np.einsum("uh,uhf->hf", del_, Yh)
    da_dst = np.einsum("vh,vhf->hf", der, Yh[:n_dst])
    dW = dY.reshape(len(x), dp).T @ x
    db = np.asarray(g, np.float64).sum(axis=0)
    return dW, da_src, da_dst, db


def forward_aggfirst(indptr, indices, x_src, n_dst, W, a_src, a_dst, b, heads, relu=True, dtype="f32", snp=None):
    """The same layer re-associated: w~_src^h = W^hT a_src^h, el_u = x_u . w~_src^h
    (and er likewise), Z_v^h = sum_u alpha_vu^h x_u, pre_v^h = W^h Z_v^h + b^h.
    dtype "bf16" rounds Z^h and W to bf16 (the CUDA path's rounding points); the
    scores use the fp32 master W.  Returns pre, alpha, Z [n_dst x H x d].

    snp = (part_of_src, C): the layer as SNP computes it (P:126 -- each source
    partition c aggregates only its own sources of v; reading G5): partition c's
    softmax over its edges (max m_c, sum S_c), its normalised partial
    Z_c^h = sum_{u in c} e^{e_vu - m_c} x_u / S_c (rounded in bf16 mode), projected,
    and the partials merged with weights w_c = S_c e^{m_c - m} / sum_c' S_c' e^{m_c' - m}
    (m = max_c m_c).  In exact arithmetic this equals the plain layer (tested)."""
    W = np.asarray(W, np.float64)
    H = heads
    dp, d = W.shape
    F = dp // H
    x = np.asarray(x_src, np.float64)
    Wh = W.reshape(H, F, d)
    ws = np.einsum("hfd,hf->hd", Wh, np.asarray(a_src, np.float64))
    wd = np.einsum("hfd,hf->hd", Wh, np.asarray(a_dst, np.float64))
    el = x @ ws.T
    er = x[:n_dst] @ wd.T
    rows, _ = _rows(indptr)
    s = el[indices] + er[rows]
    alpha = edge_softmax(indptr, _leaky(s))
    Wp = bf16_round(Wh) if dtype == "bf16" else Wh
    if snp is not None:
        part, C = snp
        e = _leaky(s)
        owner = np.asarray(part)[indices]
        parts_m = np.full((C, n_dst, H), -np.inf)
        for c in range(C):
            sel = owner == c
            np.maximum.at(parts_m[c], rows[sel], e[sel])
        m = parts_m.max(axis=0)
        Q = np.zeros((n_dst, H, F))
        wsum = np.zeros((n_dst, H))
        for c in range(C):
            sel = owner == c
            mc = parts_m[c]
            p = np.exp(e[sel] - mc[rows[sel]])
            Sc = np.zeros((n_dst, H))
            np.add.at(Sc, rows[sel], p)
            Zc = np.zeros((n_dst, H, d))
            np.add.at(Zc, rows[sel], p[:, :, None] * x[indices[sel]][:, None, :])
            Zc = np.where(Sc[:, :, None] > 0, Zc / np.where(Sc > 0, Sc, 1.0)[:, :, None], 0.0)
            if dtype == "bf16":
                Zc = bf16_round(Zc)
            wc = np.where(Sc > 0, Sc * np.exp(np.where(Sc > 0, mc - m, 0.0)), 0.0)
            Q += wc[:, :, None] * np.einsum("vhd,hfd->vhf", Zc, Wp)
            wsum += wc
        Q = np.where(wsum[:, :, None] > 0, Q / np.where(wsum > 0, wsum, 1.0)[:, :, None], 0.0)
        pre = Q.reshape(n_dst, dp) + np.asarray(b, np.float64)
        h = np.maximum(pre, 0.0) if relu else pre
        return {"pre": pre, "h": h, "alpha": alpha, "Z": None, "s": s}
    Z = np.zeros((n_dst, H, d))
    np.add.at(Z, rows, alpha[:, :, None] * x[indices][:, None, :])
    if dtype == "bf16":
        Z = bf16_round(Z)
    pre = np.einsum("vhd,hfd->vhf", Z, Wp).reshape(n_dst, dp) + np.asarray(b, np.float64)
    h = np.maximum(pre, 0.0) if relu else pre
    return {"pre": pre, "h": h, "alpha": alpha, "Z": Z, "s": s}
