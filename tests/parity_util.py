"""Tolerances of the parity tests (BASELINE.json north_star).

Every floating-point comparison is elementwise, |got - ref| <= rtol |ref| + atol, with
rtol the north star's (fp32 1e-5, bf16 2e-2) and atol = LAMBDA sigma: the spread the
definition itself admits between two correct evaluations (readings T1-T3, DESIGN.md
§13), derived from the oracle's own fp64 intermediates by propagating error VARIANCES
(probabilistic rounding-error analysis, Higham & Mary 2019: independent, mean-zero
rounding errors, each |delta| <= u |x|):

T1  fp32 accumulation order: an n-term fp32 sum of any order has error std
    <= sqrt(n) u32 sum|terms|.  fp32 mode keeps the north star's atol 1e-6 as a floor.
T2  bf16 rounding points (Z, W, hidden H, the backward's G and dZ/deg: readings R4,
    R11, R13): a point the oracle does not emulate adds variance (u_b x)^2, u_b = 2^-9;
    a point it does emulate rounds both sides identically unless their fp32 / fp64
    inputs straddle a rounding midpoint -- probability ~ 2 sigma_in / ulp, error one ulp
    -- which adds variance 4 u_b |x| sigma_in.  Variances propagate through the linear
    maps (W, the mean, its adjoint, the CE gradient's softmax Jacobian); where one error
    feeds several rows (a source row read by r destinations, a destination's dZ pulled
    into its deg sources) its variance is multiplied by that count (Cauchy-Schwarz:
    (sum_k a_k)^2 <= c sum_k a_k^2), so later sums over rows stay covered.
T3  ReLU masks are floating-point decisions: where |pre| <= LAMBDA sigma_pre either bit
    is correct (several results are correct).  `adopt_masks` checks that every mask bit
    the GPU took differently from the oracle lies in that band, then re-runs the oracle's
    backward (oracle/model.py, unchanged) with the GPU's bit at exactly those elements,
    so the gradients are compared under the same, valid, decisions.
LAMBDA = 6: a Gaussian 6-sigma tail is 2e-9 per element, below one expected false
alarm over the ~1e8 elements the suite compares.
"""
import numpy as np

import oracle

U32 = 2.0 ** -24
UB = 2.0 ** -9
LAMBDA = 6.0


def t1(abs_a, abs_b, n):
    """T1 atol of an fp32-accumulated product A @ B of n-term sums: LAMBDA sqrt(n) u32 (|A| @ |B|)."""
    return LAMBDA * np.sqrt(max(int(n), 1)) * U32 * (abs_a @ abs_b)


def rms(x):
    x = np.asarray(x, np.float64)
    return float(np.sqrt(np.mean(x ** 2))) if x.size else 0.0


def _emul(var_in, x):
    """Variance after an EMULATED rounding point (T2): one-ulp flips with probability
    ~ 2 sigma_in / ulp(x), capped at one ulp everywhere."""
    return var_in + np.minimum(4 * UB * np.abs(x) * np.sqrt(var_in), (2 * UB * x) ** 2)


def error_bounds(blocks, params, ref, mode, n_global):
    """atol arrays (LAMBDA sigma, T1-T3) for every layer's H and every dW / db.

    blocks: the oracle's blocks (hop 0 at the seeds); params: [(W, b)] the step used;
    ref: model.train_step's output for the same step (rounded or unrounded per mode);
    mode: "f32", "bf16" (vs the rounding-emulating oracle) or "bf16u" (vs the unrounded
    fp64 definition); n_global: the loss normaliser (Z20).  Returns dict(H=[K], dW=[K],
    db=[K])."""
    K = len(blocks)
    cache, gs = ref["cache"], ref["g"]
    Ws = [np.asarray(W, np.float64) for W, _ in params]
    if mode != "f32":
        Wr = [oracle.bf16_round(W) for W in Ws]
    else:
        Wr = Ws
    W2 = [W ** 2 for W in Wr]
    unr = mode == "bf16u"
    bf = mode != "f32"

    def acc2(X2, W2_, n):       # T1: fp32 accumulation variance of X W^T
        return n * U32 ** 2 * (np.sqrt(X2) @ np.sqrt(W2_).T) ** 2

    def inv_deg(blk):
        d = np.diff(blk.indptr).astype(np.float64)
        return np.where(d > 0, 1.0 / np.maximum(d, 1), 0.0)[:, None]

    VP, VH, VZ, SIG_PRE = [], [], [], []
    for l in range(1, K + 1):
        blk = blocks[K - l]
        Zs = cache["Zparts"] if (l == 1 and cache["Zparts"] is not None) else [cache["Z"][l - 1]]
        if l == 1:
            vz = sum((UB * z) ** 2 for z in Zs) if unr else np.zeros_like(Zs[0])   # Z1 exact under O4
        else:
            # a source row's error enters every destination row that reads it: Cauchy-Schwarz
            # factor r_u (its reader count) covers any later linear combination of those rows
            r_u = np.bincount(blk.indices, minlength=blk.n_src).astype(np.float64)[:, None]
            vz = oracle.aggregate(blk.indptr, blk.indices, VH[-1] * r_u) * inv_deg(blk)
            z = cache["Z"][l - 1]
            vz = vz + (UB * z) ** 2 if unr else (_emul(vz, z) if bf else vz)
        Z2 = sum(z ** 2 for z in Zs)
        vp = vz @ W2[l - 1].T + acc2(Z2, W2[l - 1], Ws[l - 1].shape[1])
        if unr:
            vp = vp + UB ** 2 * (Z2 @ W2[l - 1].T)                     # W rounding
        pre, h = cache["pre"][l - 1], cache["h"][l - 1]
        sp = np.sqrt(vp)
        if l < K:
            vh = np.where(pre > -LAMBDA * sp, vp, 0.0)                 # ReLU is 1-Lipschitz
            vh = vh + (UB * h) ** 2 if unr else (_emul(vh, h) if bf else vh)
        else:
            vh = vp
        VZ.append(vz)
        VP.append(vp)
        VH.append(vh)
        SIG_PRE.append(sp)
    # backward: g_K = (softmax - onehot) / N
    N = float(n_global)
    logits = cache["logits"]
    p = np.exp(logits - logits.max(axis=1, keepdims=True))
    p /= p.sum(axis=1, keepdims=True)
    vl = VH[K - 1]
    VG = [None] * K
    VG[K - 1] = p ** 2 * (vl + (p ** 2 * vl).sum(axis=1, keepdims=True)) / N ** 2
    for l in range(K, 0, -1):
        g = gs[l - 1]
        if bf:
            VG[l - 1] = VG[l - 1] + (UB * g) ** 2                      # R4: G rounded for tcgen05
        if l == 1:
            break
        blk = blocks[K - l]
        W = Ws[l - 1]
        dZ = g @ Wr[l - 1]
        vdz = VG[l - 1] @ W2[l - 1] + acc2(g ** 2, W2[l - 1].T, W.shape[0])
        if unr:
            vdz = vdz + UB ** 2 * ((g ** 2) @ W2[l - 1])
        if bf:
            vdz = vdz + (UB * dZ) ** 2                                  # R13: dZ / deg rounded
        # dZ[v]/deg(v) enters deg(v) source rows: variance (vdz/deg^2) x Cauchy-Schwarz factor deg
        vdh = oracle.aggregate_bwd(blk.indptr, blk.indices, vdz, blk.n_src)
        pre = cache["pre"][l - 2]
        VG[l - 2] = np.where(pre > 0, vdh, 0.0)
    out = {"H": [LAMBDA * np.sqrt(v) for v in VH], "dW": [], "db": [], "sig_pre": SIG_PRE}
    for l in range(1, K + 1):
        Zs = cache["Zparts"] if (l == 1 and cache["Zparts"] is not None) else [cache["Z"][l - 1]]
        Z2 = sum(z ** 2 for z in Zs)
        Zabs = sum(np.abs(z) for z in Zs)
        g = gs[l - 1]
        n = g.shape[0]
        # G's and Z's errors in one row may be correlated: (a + b)^2 <= 2 a^2 + 2 b^2
        vdw = 2 * (VG[l - 1].T @ Z2 + (g ** 2).T @ VZ[l - 1]) + n * U32 ** 2 * (np.abs(g).T @ Zabs) ** 2
        vdb = VG[l - 1].sum(axis=0) + n * U32 ** 2 * np.abs(g).sum(axis=0) ** 2
        out["dW"].append(LAMBDA * np.sqrt(vdw))
        out["db"].append(LAMBDA * np.sqrt(vdb))
    return out


def adopt_masks(blocks, ref, H_gpu, bounds, lr=None, params=None):
    """T3: the GPU's ReLU mask bits where they differ from the oracle's must all lie in
    the ambiguity band |pre| <= LAMBDA sigma_pre; the oracle's backward is then re-run
    with those bits (returns a new train_step-like dict; the forward is unchanged).
    H_gpu: the GPU's hidden activations, layers 1..K-1 (H > 0 <=> mask on)."""
    from oracle import model
    K = len(blocks)
    cache = dict(ref["cache"])
    pres = [np.array(p, np.float64, copy=True) for p in cache["pre"]]
    flips = []
    for l in range(1, K):
        on_g = np.asarray(H_gpu[l - 1]) > 0
        on_r = pres[l - 1] > 0
        d = on_g != on_r
        amb = np.abs(pres[l - 1]) <= LAMBDA * bounds["sig_pre"][l - 1]
        bad = d & ~amb
        assert not bad.any(), (f"layer {l}: {int(bad.sum())} ReLU mask bits differ from the oracle outside the "
                               f"ambiguity band (e.g. pre {pres[l - 1][bad][:4]}, sigma "
                               f"{bounds['sig_pre'][l - 1][bad][:4]})")
        pres[l - 1][d] = np.where(on_g[d], 1e-300, -1e-300)
        flips.append(int(d.sum()))
    cache["pre"] = pres
    grads, gs = model.backward(blocks, cache, ref["g"][K - 1])
    out = dict(ref, cache=cache, grads=grads, g=gs, mask_flips=flips)
    if lr is not None:
        out["new_params"] = [(np.asarray(W, np.float64) - lr * dW, np.asarray(b, np.float64) - lr * db)
                             for (W, b), (dW, db) in zip(params, grads)]
    return out


def reconcile(blocks, params, ref, mode, n_global, H_gpu):
    """error_bounds + adopt_masks: returns (ref with the GPU's valid mask bits, bounds)."""
    bd = error_bounds(blocks, params, ref, mode, n_global)
    ref = adopt_masks(blocks, ref, H_gpu, bd)
    return ref, error_bounds(blocks, params, ref, mode, n_global)


def sum_bounds(bounds):
    """Bounds of an all-reduced gradient: the sum over ranks of every rank's bound."""
    out = {"dW": [], "db": []}
    K = len(bounds[0]["dW"])
    for l in range(K):
        out["dW"].append(sum(b["dW"][l] for b in bounds))
        out["db"].append(sum(b["db"][l] for b in bounds))
    return out


def assert_close(got, ref, dtype, what, bound=None):
    """|got - ref| <= rtol |ref| + atol elementwise.  fp32: rtol 1e-5, atol max(1e-6, bound);
    bf16: rtol 2e-2, atol = bound (T1-T3) or, with no bound given, 2e-2 rms(ref);
    "bf16u" (vs the unrounded definition): atol = max(bound, 2e-2 rms(ref)) (reading T4:
    the bf16 copy of W shifts every row by the same rounding error, which the variance
    model treats as independent; the normwise floor covers that shared shift)."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    assert got.shape == ref.shape, (what, got.shape, ref.shape)
    if dtype == "f32":
        rtol = 1e-5
        atol = np.maximum(1e-6, bound) if bound is not None else 1e-6
    elif dtype == "bf16u":
        rtol = 2e-2
        atol = np.maximum(bound, 2e-2 * rms(ref)) if bound is not None else 2e-2 * rms(ref)
    else:
        rtol = 2e-2
        atol = bound if bound is not None else 2e-2 * rms(ref)
    err = np.abs(got - ref)
    lim = atol + rtol * np.abs(ref)
    bad = err > lim
    if bad.any():
        i = np.unravel_index(np.argmax(err - lim), ref.shape)
        raise AssertionError(f"{what}: {int(bad.sum())}/{ref.size} elements outside the bar (worst at {i}: got "
                             f"{got[i]!r} ref {ref[i]!r} allowed {np.broadcast_to(lim, ref.shape)[i]!r}; max abs "
                             f"err {err.max():.3e}, ref rms {rms(ref):.3e})")


def gat_bounds(indptr, indices, x_src, n_dst, W, a_src, a_dst, b, cache, g, heads, dtype):
    """atol of the GAT layer's h, dW, db, da_src, da_dst (reading T5): the
    layer's forward and backward (oracle/gat.py) re-evaluated on MAGNITUDES -- every
    signed sum replaced by the sum of the absolute values of its terms, the softmax
    Jacobian by its absolute bound alpha (|d| + sum alpha |d|) -- gives M, the size of
    the terms behind every output; a first-order bound is then c u M: fp32 (T1, the
    longest sum is over the n_src sources) c = LAMBDA (sqrt(n_src) + 8), u = 2^-24; bf16
    (T2: W, Z, g, gamma rounded along the chain) c = 4, u = 2^-8."""
    W = np.abs(np.asarray(W, np.float64))
    H = heads
    dp, d = W.shape
    F = dp // H
    x = np.abs(np.asarray(x_src, np.float64))
    n_src = x.shape[0]
    rows = np.repeat(np.arange(n_dst), np.diff(indptr))
    alpha = cache["alpha"]
    Ya = (x @ W.T).reshape(n_src, H, F)
    As = np.abs(np.asarray(a_src, np.float64)).reshape(H, F)
    Ad = np.abs(np.asarray(a_dst, np.float64)).reshape(H, F)
    el = np.einsum("uhf,hf->uh", Ya, As)
    er = np.einsum("uhf,hf->uh", Ya[:n_dst], Ad)
    sm = el[indices] + er[rows]                                  # |score| terms per edge
    smax = np.zeros((n_dst, H))
    np.maximum.at(smax, rows, sm)
    agg = np.zeros((n_dst, H, F))
    np.add.at(agg, rows, alpha[:, :, None] * Ya[indices])
    Mh = (agg * (1.0 + 2.0 * smax[:, :, None])).reshape(n_dst, dp) + np.abs(np.asarray(b, np.float64))
    gm = np.abs(np.asarray(g, np.float64)).reshape(n_dst, H, F)
    dal = np.einsum("ehf,ehf->eh", gm[rows], Ya[indices])
    t = np.zeros((n_dst, H))
    np.add.at(t, rows, alpha * dal)
    de = alpha * (dal + t[rows])
    dY = np.zeros((n_src, H, F))
    np.add.at(dY, indices, alpha[:, :, None] * gm[rows])
    dl = np.zeros((n_src, H))
    np.add.at(dl, indices, de)
    dr = np.zeros((n_dst, H))
    np.add.at(dr, rows, de)
    dY += dl[:, :, None] * As[None]
    dY[:n_dst] += dr[:, :, None] * Ad[None]
    Mda_s = np.einsum("uh,uhf->hf", dl, Ya).reshape(-1)
    Mda_d = np.einsum("vh,vhf->hf", dr, Ya[:n_dst]).reshape(-1)
    MdW = dY.reshape(n_src, dp).T @ x
    Mdb = gm.reshape(n_dst, dp).sum(axis=0)
    cu = LAMBDA * (np.sqrt(n_src) + 8) * U32 if dtype == "f32" else 4 * 2.0 ** -8
    return {"h": cu * Mh, "dW": cu * MdW, "db": cu * Mdb, "da_src": cu * Mda_s, "da_dst": cu * Mda_d}
