"""Per-rank emulation of APT's four strategies + the Eq. 2 cost model -- ORACLE.

TEST INFRASTRUCTURE ONLY.  Emulates C ranks in one process:
it builds, for each strategy, exactly what every rank owns, sends and reads for
the first GNN layer, and counts the paper's quantities N_d, N_vs, N_vd
 plus the exact bytes of the message formats DESIGN.md §Messages
fixes.  The numerical result of every strategy is the 1-GPU result (P:59,
P:279 "semantically equivalent"), so h^1 / dW are compared against
``oracle.model`` on the same global batch; this module pins the *structures*.

Strategies (Fig. 3; Fig. 5 P:219 tensor partitioning):
  GDP  seeds split by chunk; each rank aggregates its own blocks; remote rows
       are read from the owning rank.
  NFP  features split by column (d/C each); every rank receives every layer-1
       block (AllBroadcast), computes partial projections of its
       column slice and sends them to the requester.
  SNP  edge-cut partition; rank c aggregates the sources it owns for every
       destination that has >=1 sampled source in partition c, a virtual node
       on c when c != requester; partial embeddings return to the requester
       (P:126).
  DNP  each layer-1 destination goes to its owning rank, which computes the
       complete h^1 and sends it back.
"""
from __future__ import annotations

import numpy as np

STRATEGIES = ("GDP", "NFP", "SNP", "DNP")

# Bandwidth-profile operator slots (DESIGN.md §Cost model; apt.h apt_bw_profile).
OP_LOCAL_GATHER, OP_PEER_PULL, OP_PEER_PUSH, OP_ALLTOALLV, OP_ALLGATHER, OP_REDUCE_SCATTER, \
    OP_ALLREDUCE, OP_HOST_GATHER = range(8)


def col_range(c, C, d):
    """NFP column slice of rank c: [floor(c*d/C), floor((c+1)*d/C))."""
    return (c * d) // C, ((c + 1) * d) // C


def assign_seeds(strategy, gbatch, part, C, B):
    """O1 / Z19: GDP, NFP take contiguous chunk r of the global batch; SNP, DNP take
    the seeds of their own partition, in permutation order (P:163 last sentence)."""
    gbatch = np.asarray(gbatch, np.int64)
    if strategy in ("GDP", "NFP"):
        return [gbatch[r * B:(r + 1) * B] for r in range(C)]
    p = part[gbatch]
    return [gbatch[p == r] for r in range(C)]


def msg_bytes_graph(G, n_e):
    """Packed sub-graph message: header(2) + row_tag[G] + deg[G]
    + indptr[G+1] + src_gid[n_e], all int32."""
    return 4 * (2 + G + G + (G + 1) + n_e)


def msg_bytes_ids(G):
    """DNP request message: header(2) + row_tag[G] + dst_gid[G], int32."""
    return 4 * (2 + 2 * G)


def _edges(blk):
    """(row, src_gid) for every edge of a block."""
    rows = np.repeat(np.arange(blk.n_dst), np.diff(blk.indptr))
    return rows, blk.src[blk.indices]


def tiered_store(part, C, hbm_frac, hot_ids=None, cache_rows=0):
    """The unified feature store's tiers (apt_fstore_create_tiered):
    every partition keeps its first ceil(hbm_frac * size) rows (ascending id) in its
    owner's HBM, the rest in the host tier; rank r replicates the first cache_rows hot
    ids it does not hold in its own HBM (excess cache).
    Returns tier(r, ids) -> array of 0 local, 1 NVLink peer, 2 host."""
    part = np.asarray(part)
    n = len(part)
    host = np.zeros(n, bool)
    for o in range(C):
        ids = np.nonzero(part == o)[0]
        keep = min(len(ids), int(np.ceil(hbm_frac * len(ids))))
        host[ids[keep:]] = True
    cached = [np.zeros(n, bool) for _ in range(C)]
    if hot_ids is not None and cache_rows:
        for r in range(C):
            taken = 0
            for u in hot_ids[:cache_rows]:
                if taken >= cache_rows:
                    break
                if (part[u] == r and not host[u]) or cached[r][u]:
                    continue
                cached[r][u] = True
                taken += 1

    def tier(r, ids):
        ids = np.asarray(ids, np.int64)
        t = np.where(part[ids] == r, 0, 1)
        t = np.where(host[ids], 2, t)
        return np.where(cached[r][ids], 0, t)
    return tier


def cache_sets(strategy, counts, part, C, budget, indptr=None, indices=None):
    """P:163 "Cache configuration": the node ids each GPU keeps in its memory, from the
    dry-run access frequencies `counts` (apt_access_counts, reading R12):
      GDP, NFP -- "the most popular nodes" (of the whole graph);
      SNP      -- "the most popular nodes in its assigned graph partition";
      DNP      -- the most popular among "the nodes in its partition and their 1-hop
                  neighbors" (needs the CSR).
    Popularity order: count descending, then id ascending (reading C1); at most `budget`
    ids per GPU.  Returns [ids of rank r, hottest first] for r in 0..C-1."""
    counts = np.asarray(counts, np.int64)
    part = np.asarray(part)
    n = len(counts)
    order = np.lexsort((np.arange(n), -counts))            # count desc, id asc
    out = []
    for r in range(C):
        if strategy in ("GDP", "NFP"):
            cand = np.ones(n, bool)
        elif strategy == "SNP":
            cand = part == r
        elif strategy == "DNP":
            own = part == r
            cand = own.copy()
            for u in np.nonzero(own)[0]:
                cand[indices[indptr[u]:indptr[u + 1]]] = True
        else:
            raise ValueError(strategy)
        out.append(order[cand[order]][:budget].astype(np.int64))
    return out


def cached_store(sets, n):
    """The unified store of P:163 caches (P:241-247 feature map): rank r reads u from
    its own cache if u is in sets[r], else from the lowest peer whose cache holds it
    (NVLink), else from the host.  Returns tier(r, ids) -> 0 local, 1 peer, 2 host."""
    C = len(sets)
    mine = [np.zeros(n, bool) for _ in range(C)]
    for r in range(C):
        mine[r][np.asarray(sets[r], np.int64)] = True
    anyc = np.any(mine, axis=0) if C else np.zeros(n, bool)

    def tier(r, ids):
        ids = np.asarray(ids, np.int64)
        return np.where(mine[r][ids], 0, np.where(anyc[ids], 1, 2))
    return tier


def emulate_layer1(strategy, l1_blocks, part, C, d, d_out, feat_bytes=4, hidden_bytes=4, tier=None, heads=0):
    """l1_blocks[r] = rank r's layer-1 Block (dst, src, indptr, indices).  tier(r, ids):
    where rank r reads each row (0 local HBM, 1 NVLink peer, 2 host; default: own
    partition local, others peer).  heads > 0: a GAT first layer, whose attention
    adds exchanges for NFP and SNP (reading G6): NFP reduces and
    reads back the partial score and dalpha of every edge of every other block
    (attn_bytes = 4 passes x H x 4 B per edge); SNP ships (m, S) with each virtual
    node's partial and (t, L) with its gradient (2H x 4 B each way), and every owner
    reads the destination's own feature row of each item it computes
    (attn_feat_bytes).  Returns per-rank dict of counts and structures."""
    if tier is None:
        def tier(r, ids):
            return np.where(np.asarray(part)[np.asarray(ids, np.int64)] == r, 0, 1)
    out = []
    N_d = [b.n_dst for b in l1_blocks]
    for r in range(C):
        out.append(dict(n_d=N_d[r], n_vs=0, n_vd=0, rows_local=0, rows_peer=0, rows_host=0,
                        feat_bytes_local=0, feat_bytes_peer=0, feat_bytes_host=0, graph_bytes=0,
                        hidden_bytes_fwd=0, hidden_bytes_bwd=0, n_calls=0, attn_bytes=0, attn_feat_bytes=0,
                        virtual=[], requests=[]))

    def count(o, uu, rec):
        t = tier(o, uu) if len(uu) else np.zeros(0, int)
        for key, code in (("local", 0), ("peer", 1), ("host", 2)):
            rec["rows_" + key] = int((t == code).sum())
            rec["feat_bytes_" + key] = rec["rows_" + key] * d * feat_bytes

    if strategy == "GDP":
        for r, blk in enumerate(l1_blocks):
            _, u = _edges(blk)
            count(r, np.unique(u), out[r])
        return out
    if strategy == "NFP":
        for c in range(C):
            lo, hi = col_range(c, C, d)
            rows = 0
            for b, blk in enumerate(l1_blocks):
                _, u = _edges(blk)
                rows += len(np.unique(u))
                if b != c:
                    out[c]["graph_bytes"] += msg_bytes_graph(blk.n_dst, blk.n_edges)
                    out[c]["hidden_bytes_bwd"] += blk.n_dst * d_out * hidden_bytes
                    if heads and C > 1:
                        out[c]["attn_bytes"] += 4 * heads * 4 * blk.n_edges
            out[c]["rows_local"] = rows
            out[c]["feat_bytes_local"] = rows * (hi - lo) * feat_bytes
            out[c]["hidden_bytes_fwd"] = (C - 1) * N_d[c] * d_out * hidden_bytes
            out[c]["n_calls"] = 3 if C > 1 else 0   # graph all-gather, partial reduce, g all-gather
        return out
    if strategy == "SNP":
        # groups[c] = list of (requester r, row v, [src gids in partition c])
        recv_rows = [set() for _ in range(C)]
        for r, blk in enumerate(l1_blocks):
            rows, u = _edges(blk)
            pu = part[u]
            for c in range(C):
                m = pu == c
                if not m.any():
                    continue
                vs = np.unique(rows[m])
                recv_rows[c].update(u[m].tolist())
                if heads and C > 1:
                    out[c]["attn_feat_bytes"] += len(vs) * d * feat_bytes
                if c != r:
                    if heads:
                        out[r]["attn_bytes"] += len(vs) * 2 * heads * 4
                        out[c]["attn_bytes"] += len(vs) * 2 * heads * 4
                    out[r]["n_vs"] += len(vs)
                    out[r]["virtual"].append((c, blk.dst[vs]))
                    out[c]["graph_bytes"] += msg_bytes_graph(len(vs), int(m.sum()))
                    out[r]["hidden_bytes_fwd"] += len(vs) * d_out * hidden_bytes
                    out[c]["hidden_bytes_bwd"] += len(vs) * d_out * hidden_bytes
        for c in range(C):
            count(c, np.fromiter(recv_rows[c], np.int64, len(recv_rows[c])), out[c])   # own partition: HBM or host
            out[c]["n_calls"] = 3 if C > 1 else 0   # graph all-to-all, partial reduce, g all-to-all
        return out
    if strategy == "DNP":
        owned_rows = [set() for _ in range(C)]   # sources read by owner o
        for r, blk in enumerate(l1_blocks):
            rows, u = _edges(blk)
            owner = part[blk.dst]
            for o in range(C):
                vs = np.nonzero(owner == o)[0]
                if len(vs) == 0:
                    continue
                m = np.isin(rows, vs)
                owned_rows[o].update(u[m].tolist())
                if o != r:
                    out[r]["n_vd"] += len(vs)
                    out[r]["requests"].append((o, blk.dst[vs]))
                    out[o]["graph_bytes"] += msg_bytes_ids(len(vs))
                    out[r]["hidden_bytes_fwd"] += len(vs) * d_out * hidden_bytes
                    out[o]["hidden_bytes_bwd"] += len(vs) * d_out * hidden_bytes
        for o in range(C):
            count(o, np.fromiter(owned_rows[o], np.int64, len(owned_rows[o])), out[o])
            out[o]["n_calls"] = 3 if C > 1 else 0   # request all-to-all, h1 return, g return
        return out
    raise ValueError(strategy)


def paper_volume(strategy, stats, d_out, hidden_bytes=4):
    """The paper's closed-form T_shuffle volumes, per rank:
    NFP 2 d' C N_d, SNP 2 d' N_vs, DNP 2 d' N_vd, GDP 0 (elements x bytes, Z14)."""
    C = len(stats)
    if strategy == "GDP":
        return [0] * C
    if strategy == "NFP":
        return [2 * d_out * C * s["n_d"] * hidden_bytes for s in stats]
    if strategy == "SNP":
        return [2 * d_out * s["n_vs"] * hidden_bytes for s in stats]
    return [2 * d_out * s["n_vd"] * hidden_bytes for s in stats]


def predict(per_strategy_stats, alpha, beta, t_build):
    """Eq. 2 minus the common T_train: for every strategy and rank
    T = T_build + T_load + T_shuffle, with T_load = bytes/beta per tier and
    T_shuffle = sum over ops (alpha * calls + bytes / beta)  (reading Z23 adds alpha).
    per_strategy_stats[s][r] are counts summed over the dry-run epoch; t_build[s][r]
    is the measured build time.  Predicted time = max over ranks (Z13).
    Returns (pred[4], pick index)."""
    pred = []
    for si, s in enumerate(STRATEGIES):
        worst = 0.0
        for r, st in enumerate(per_strategy_stats[si]):
            steps = st.get("steps", 1)
            t = t_build[si][r]
            t += st["feat_bytes_local"] / beta[OP_LOCAL_GATHER] + steps * alpha[OP_LOCAL_GATHER]
            if st["feat_bytes_peer"]:
                t += st["feat_bytes_peer"] / beta[OP_PEER_PULL] + steps * alpha[OP_PEER_PULL]
            if st.get("feat_bytes_host"):   # host tier of the unified store
                t += st["feat_bytes_host"] / beta[OP_HOST_GATHER] + steps * alpha[OP_HOST_GATHER]
            if s == "NFP" and st["n_calls"]:
                t += 2 * steps * alpha[OP_ALLGATHER] + steps * alpha[OP_REDUCE_SCATTER]
                t += st["graph_bytes"] / beta[OP_ALLGATHER]
                t += st["hidden_bytes_fwd"] / beta[OP_REDUCE_SCATTER]
                t += st["hidden_bytes_bwd"] / beta[OP_ALLGATHER]
                if st.get("attn_bytes", 0) > 0:    # GAT: partial scores / dalpha all-reduced
                    t += 2 * steps * alpha[OP_ALLREDUCE] + st["attn_bytes"] / beta[OP_ALLREDUCE]
            elif s in ("SNP", "DNP") and st["n_calls"]:
                t += 3 * steps * alpha[OP_ALLTOALLV]
                t += (st["graph_bytes"] + st["hidden_bytes_fwd"] + st["hidden_bytes_bwd"]
                      + st.get("attn_bytes", 0)) / beta[OP_ALLTOALLV]
            if st.get("attn_feat_bytes"):   # SNP-GAT: destinations' own rows
                t += st["attn_feat_bytes"] / beta[OP_PEER_PULL]
            worst = max(worst, t)
        pred.append(worst)
    pick = int(np.argmin(pred))
    return pred, pick


def access_counts(graph, train, fanouts, sample_seed, epoch, C, B, n_steps):
    """Node access frequencies (Table 3; reading R12): counts[u] =
    number of (step, rank) pairs among the first n_steps global steps of the epoch, GDP
    seed split, whose layer-1 block reads u's input row, i.e. u is the source of at
    least one sampled layer-1 edge (the dst prefix is not loaded unless it is also a
    sampled neighbour)."""
    from . import epoch_perm, global_batch, sample_blocks
    perm = epoch_perm(train, sample_seed, epoch)
    counts = np.zeros(graph.n, np.int64)
    for t in range(n_steps):
        gb = global_batch(perm, t, C, B)
        for seeds in assign_seeds("GDP", gb, None, C, B):
            if len(seeds) == 0:
                continue
            blk = sample_blocks(graph, seeds, fanouts, sample_seed, t)[-1]
            counts[np.unique(blk.src[blk.indices])] += 1
    return counts


def skew_table(counts, edges=(0.01, 0.05, 0.10, 0.20, 0.50, 1.0)):
    """Table 3's access ratios: rank nodes by access count (descending) and report the
    share of all accesses that falls in each rank bucket (<1%, 1-5%, ..., 50-100%)."""
    c = np.sort(np.asarray(counts, np.int64))[::-1]
    total = max(1, int(c.sum()))
    n = len(c)
    out, lo = [], 0
    for e in edges:
        hi = int(round(e * n))
        out.append(float(c[lo:hi].sum()) / total)
        lo = hi
    return out
