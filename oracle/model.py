"""fp64 GraphSAGE forward / backward -- ORACLE (test infrastructure only).

Follows Eq. 1: h_v^k = sigma[AGG^k({W^k h_u^{k-1} : u in N(v)})] with
W^k of shape d' x d, AGG = mean (GraphSAGE), sigma = ReLU on
hidden layers and identity on the output (reading Z9), bias added once after
the aggregation (Z10), W applied after the mean (Z8: W*mean = mean(W*) in
exact arithmetic).  Loss = sum_s CE(h^K_s, y_s) / |global batch| (Z20).

bf16 mode emulates the CUDA path's rounding points (O5): features are exact
in bf16 (O4), Z -> fp32 -> bf16 RNE, W -> bf16 RNE, hidden activations
h^l (l < K) -> bf16 RNE after bias + ReLU (reading R11: the next
layer's mean and the ReLU mask read the stored bf16 copy), everything else fp64.
"""
from __future__ import annotations

import numpy as np

from . import aggregate, aggregate_bwd, bf16_round, features


def snp_partials(blk, x_src, part, C):
    """SNP's partial aggregates of layer 1:
    P~_c[v] = (1/deg_s(v)) * sum over sampled sources u of v with part(u) = c of x_u,
    one [n_dst x d] array per partition c.  sum_c P~_c = the mean (exact arithmetic)."""
    deg = np.diff(blk.indptr)
    rows = np.repeat(np.arange(blk.n_dst), deg)
    owner = np.asarray(part)[blk.src[blk.indices]]
    out = []
    for c in range(C):
        m = owner == c
        acc = np.zeros((blk.n_dst, x_src.shape[1]), np.float64)
        np.add.at(acc, rows[m], x_src[blk.indices[m]])
        out.append(np.where(deg[:, None] > 0, acc / np.maximum(deg, 1)[:, None], 0.0))
    return out


def forward(blocks, feat_seed, dim, params, dtype="f32", x0=None, snp=None):
    """params: [(W [d_out x d_in], b [d_out])] layer 1 first.  blocks[h], hop 0 at seeds.
    snp = (part, C): layer 1 is computed as SNP does -- partial aggregates P~_c, each
    rounded at the bf16 rounding point and projected, summed before bias/ReLU (Z10).
    Returns a dict with per-layer Z, pre, h (fp64) and the logits."""
    K = len(blocks)
    assert len(params) == K
    H = features(feat_seed, blocks[K - 1].src, dim) if x0 is None else np.asarray(x0, np.float64)
    cache = {"Z": [], "pre": [], "h": [], "W": [], "Zparts": None}
    for l in range(1, K + 1):
        blk = blocks[K - l]
        W, b = params[l - 1]
        W = np.asarray(W, np.float64)
        if dtype == "bf16":
            W = bf16_round(W)
        if l == 1 and snp is not None:
            parts = snp_partials(blk, H, snp[0], snp[1])
            if dtype == "bf16":
                parts = [bf16_round(P) for P in parts]
            cache["Zparts"] = parts
            Z = sum(parts)
            pre = sum(P @ W.T for P in parts) + np.asarray(b, np.float64)
        else:
            Z = aggregate(blk.indptr, blk.indices, H)
            if dtype == "bf16":
                Z = bf16_round(Z)
            pre = Z @ W.T + np.asarray(b, np.float64)
        H = np.maximum(pre, 0.0) if l < K else pre
        if dtype == "bf16" and l < K:
            H = bf16_round(H)                  # reading R11
        cache["Z"].append(Z)
        cache["pre"].append(pre)
        cache["h"].append(H)
        cache["W"].append(W)
    cache["logits"] = H
    return cache


def ce_loss_grad(logits, labels, n_global):
    """Cross entropy summed over the seeds / n_global (Z20) and d loss / d logits."""
    m = logits.max(axis=1, keepdims=True)
    e = np.exp(logits - m)
    s = e.sum(axis=1, keepdims=True)
    logp = logits - m - np.log(s)
    idx = np.arange(len(labels))
    loss = -logp[idx, labels].sum() / n_global
    g = e / s
    g[idx, labels] -= 1.0
    return loss, g / n_global


def backward(blocks, cache, g_logits):
    """Returns [(dW_l, db_l)] layer 1 first, plus per-layer g (= dL/dpre)."""
    K = len(blocks)
    grads = [None] * K
    gs = [None] * K
    g = g_logits
    for l in range(K, 0, -1):
        Z = cache["Z"][l - 1]
        W = cache["W"][l - 1]
        gs[l - 1] = g
        if l == 1 and cache.get("Zparts") is not None:
            grads[l - 1] = (sum(g.T @ P for P in cache["Zparts"]), g.sum(axis=0))
        else:
            grads[l - 1] = (g.T @ Z, g.sum(axis=0))
        if l > 1:
            blk = blocks[K - l]
            dZ = g @ W
            dH = aggregate_bwd(blk.indptr, blk.indices, dZ, blk.n_src)
            g = dH * (cache["pre"][l - 2] > 0)
    return grads, gs


def train_step(blocks, feat_seed, dim, params, labels_of_seeds, n_global, dtype="f32", lr=None, snp=None):
    cache = forward(blocks, feat_seed, dim, params, dtype, snp=snp)
    loss, g = ce_loss_grad(cache["logits"], labels_of_seeds, n_global)
    grads, gs = backward(blocks, cache, g)
    out = {"loss": loss, "cache": cache, "grads": grads, "g": gs}
    if lr is not None:
        out["new_params"] = [(np.asarray(W, np.float64) - lr * dW, np.asarray(b, np.float64) - lr * db)
                             for (W, b), (dW, db) in zip(params, grads)]
    return out
