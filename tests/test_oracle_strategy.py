"""Pins for the oracle's strategy emulation and cost model (-m "not gpu").

The worked example of Figs. 2-3 pins the virtual-node / remote-row
logic; closed-form volumes pin the counters; Table 1's text
 gives directional checks.
"""
import os

import numpy as np
import pytest

import aptgen
import oracle
from oracle import strategy as S

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig2_fig3_example.txt")


def _golden():
    """tests/golden/fig2_fig3_example.txt: the paper's Fig. 2/3 example."""
    part, blocks, expect = {}, {}, []
    for line in open(GOLDEN):
        w = line.split()
        if not w or w[0].startswith("#"):
            continue
        if w[0] == "partition":
            part.update({c: int(w[1][3:]) - 1 for c in w[2:]})
        elif w[0] == "block":
            blocks.setdefault(int(w[1][3:]) - 1, []).append((w[2], w[4:]))
        elif w[0] == "expect":
            expect.append(w[1:])
    return part, blocks, expect


# Fig. 2(a)/3 node names -> ids.  GPU 1 manages A,B,E,G,H; GPU 2 manages C,D,F,M,K.
_PART, _BLOCKS, _EXPECT = _golden()
NAMES = "".join(sorted(_PART))
ID = {c: i for i, c in enumerate(NAMES)}
PART = np.array([_PART[c] for c in NAMES], np.int32)


def hand_block(dst, edges):
    """Hand-built layer-1 block (no sampler): dst list, {dst: [src...]}."""
    dst_ids = np.array([ID[c] for c in dst], np.int64)
    new = sorted({ID[u] for v in dst for u in edges.get(v, [])} - set(dst_ids.tolist()))
    src = np.concatenate([dst_ids, np.array(new, np.int64)])
    pos = {int(u): i for i, u in enumerate(src)}
    indptr, indices = [0], []
    for v in dst:
        us = sorted(ID[u] for u in edges.get(v, []))
        indices += [pos[u] for u in us]
        indptr.append(len(indices))
    return oracle.Block(1, dst_ids, src, np.array(indptr, np.int64), np.array(indices, np.int32),
                        None, None, 0)


@pytest.fixture
def fig2():
    # seed A on GPU 1: layer-1 destinations B, K; B <- G, H and K <- D, A.
    out = []
    for g in range(2):
        rows = _BLOCKS.get(g, [])
        out.append(hand_block("".join(v for v, _ in rows), {v: "".join(us) for v, us in rows}))
    return out


def test_fig3_golden_expectations(fig2):
    """Every `expect` line of the golden file (each cites its passage there)."""
    assert len(_EXPECT) >= 10
    for strat, key, *args in _EXPECT:
        if key == "col_range":
            assert S.col_range(int(args[0][3:]) - 1, 2, 4) == (int(args[1]), int(args[2]))
            continue
        st = S.emulate_layer1(strat, fig2, PART, 2, d=4, d_out=2)
        g = int(args[0][3:]) - 1
        if key in ("virtual", "requests", "request"):
            field = "virtual" if key == "virtual" else "requests"
            (o, vs), = st[g][field]
            assert o == int(args[1][3:]) - 1 and "".join(NAMES[v] for v in vs) == args[2], (strat, key)
        else:
            assert st[g][key] == int(args[1]), (strat, key, st[g][key])


def test_fig3_snp_one_virtual_node(fig2):
    st = S.emulate_layer1("SNP", fig2, PART, 2, d=4, d_out=2)
    assert st[0]["n_vs"] == 1                                  # K' on GPU 2 (source D)
    (c, vs), = st[0]["virtual"]
    assert c == 1 and [NAMES[v] for v in vs] == ["K"]
    assert st[1]["rows_local"] == 1                            # GPU 2 reads only D
    assert st[0]["rows_peer"] == st[1]["rows_peer"] == 0       # SNP reads are all local


def test_fig3_dnp_ships_k_and_reads_a_remotely(fig2):
    st = S.emulate_layer1("DNP", fig2, PART, 2, d=4, d_out=2)
    assert st[0]["n_vd"] == 1                                  # K -> GPU 2
    (o, vs), = st[0]["requests"]
    assert o == 1 and [NAMES[v] for v in vs] == ["K"]
    assert st[1]["rows_local"] == 1 and st[1]["rows_peer"] == 1   # D local, A remote
    assert st[0]["rows_local"] == 2 and st[0]["rows_peer"] == 0   # G, H for B


def test_fig3_nfp_gpu2_gets_latter_half_columns(fig2):
    st = S.emulate_layer1("NFP", fig2, PART, 2, d=4, d_out=2)
    assert S.col_range(1, 2, 4) == (2, 4)                      # latter-half dims
    assert st[1]["graph_bytes"] == S.msg_bytes_graph(2, 4)     # GPU 2 receives GPU 1's graph
    assert st[1]["rows_local"] == 4 and st[1]["feat_bytes_local"] == 4 * 2 * 4
    assert st[0]["hidden_bytes_fwd"] == 1 * 2 * 2 * 4          # B, K partials from GPU 2


def test_fig3_gdp_reads_d_remotely(fig2):
    st = S.emulate_layer1("GDP", fig2, PART, 2, d=4, d_out=2)
    assert st[0]["rows_peer"] == 1 and st[0]["rows_local"] == 3   # D remote; G, H, A local
    assert all(s["hidden_bytes_fwd"] == 0 for s in st)        # GDP T_shuffle = 0


def test_fig3_gat_attention_costs(fig2):
    # P:344 / P:173-178: attention costs GDP and DNP nothing extra; SNP ships the softmax
    # state with K' (1 virtual node: (m, S) out, (t, L) back) and GPU 2 reads K's own row
    # for the score; NFP sums partial scores of GPU 1's 4 edges (2 passes fwd, 2 bwd)
    H = 4
    for s in ("GDP", "DNP"):
        assert all(r["attn_bytes"] == 0 and r["attn_feat_bytes"] == 0
                   for r in S.emulate_layer1(s, fig2, PART, 2, d=4, d_out=8, heads=H))
    snp = S.emulate_layer1("SNP", fig2, PART, 2, d=4, d_out=8, heads=H)
    assert snp[0]["attn_bytes"] == snp[1]["attn_bytes"] == 1 * 2 * H * 4
    # GPU 1 computes B (G, H) and K (A) locally, GPU 2 computes K' (D): one dst row each item
    assert snp[0]["attn_feat_bytes"] == 2 * 4 * 4 and snp[1]["attn_feat_bytes"] == 1 * 4 * 4
    nfp = S.emulate_layer1("NFP", fig2, PART, 2, d=4, d_out=8, heads=H)
    assert nfp[1]["attn_bytes"] == 4 * H * 4 * 4 and nfp[0]["attn_bytes"] == 0
    sage = S.emulate_layer1("SNP", fig2, PART, 2, d=4, d_out=8)
    assert sage[0]["attn_bytes"] == 0 and sage[0]["hidden_bytes_fwd"] == snp[0]["hidden_bytes_fwd"]


def _rank_blocks(graph, cfg, C, strategy, step=0):
    train = aptgen.train_nodes(graph, cfg)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, step, C, 64)
    part = aptgen.partition(graph.n, C)
    seeds = S.assign_seeds(strategy, gb, part, C, 64)
    blocks = [oracle.sample_blocks(graph, s, cfg.fanouts, cfg.sample_seed, step)[-1] for s in seeds]
    return blocks, part, gb, seeds


@pytest.mark.parametrize("C", [2, 4, 8])
def test_volumes_equal_paper_formulas(tiny_graph, tiny_cfg, C):
    d, dd = tiny_cfg.dim, tiny_cfg.hidden
    for s in S.STRATEGIES:
        blocks, part, gb, seeds = _rank_blocks(tiny_graph, tiny_cfg, C, s)
        st = S.emulate_layer1(s, blocks, part, C, d, dd)
        counted = sum(x["hidden_bytes_fwd"] + x["hidden_bytes_bwd"] for x in st)
        paper = sum(S.paper_volume(s, st, dd))
        if s in ("GDP", "SNP", "DNP"):
            assert counted == paper                             # P:146, 148, 161 exactly
        else:
            # P:147 counts 2 d' C N_d including each rank's own partial; the wire
            # carries the (C-1) remote ones (reading Z15).
            assert counted * C == paper * (C - 1)
        assert sum(x["n_d"] for x in st) == sum(len(b.dst) for b in blocks)
        # seed assignment is a partition of the global batch
        assert np.array_equal(np.sort(np.concatenate(seeds)), np.sort(gb))


@pytest.mark.parametrize("C", [2, 4, 8])
def test_table1_directional_tradeoffs(tiny_graph, tiny_cfg, C):
    """NFP ships the most hidden embeddings, DNP at most one per dst;
    SNP/NFP read all features locally; only GDP and DNP read remote rows."""
    vol = {}
    for s in S.STRATEGIES:
        blocks, part, _, _ = _rank_blocks(tiny_graph, tiny_cfg, C, s)
        st = S.emulate_layer1(s, blocks, part, C, tiny_cfg.dim, tiny_cfg.hidden)
        vol[s] = sum(x["hidden_bytes_fwd"] for x in st)
        if s in ("SNP", "NFP"):
            assert all(x["rows_peer"] == 0 for x in st)
        if s == "DNP":
            assert all(x["n_vd"] <= x["n_d"] for x in st)
        if s == "SNP":
            assert all(x["n_vs"] <= (C - 1) * x["n_d"] for x in st)
    assert vol["GDP"] == 0
    assert vol["NFP"] >= vol["SNP"] and vol["NFP"] >= vol["DNP"]


def test_snp_dnp_degrade_under_random_partition(tiny_graph, tiny_cfg):
    """Fig. 11: a random partition raises N_vs and N_vd."""
    C = 4
    good = {}
    for part_kind in ("planted", "random"):
        for s in ("SNP", "DNP"):
            blocks, part, _, _ = _rank_blocks(tiny_graph, tiny_cfg, C, s)
            if part_kind == "random":
                part = np.random.default_rng(0).integers(0, C, tiny_graph.n).astype(np.int32)
            st = S.emulate_layer1(s, blocks, part, C, tiny_cfg.dim, tiny_cfg.hidden)
            good[(part_kind, s)] = sum(x["n_vs"] + x["n_vd"] for x in st)
    assert good[("random", "SNP")] > good[("planted", "SNP")]
    assert good[("random", "DNP")] > good[("planted", "DNP")]


def test_cost_model_picks_argmin_and_gdp_wins_when_shuffle_is_costly():
    mk = lambda **kw: [dict(dict(feat_bytes_local=0, feat_bytes_peer=0, graph_bytes=0,
                                 hidden_bytes_fwd=0, hidden_bytes_bwd=0, n_calls=3, steps=1), **kw)]
    stats = [mk(feat_bytes_local=1e9, feat_bytes_peer=1e9, n_calls=0),
             mk(feat_bytes_local=1e8, hidden_bytes_fwd=1e10, hidden_bytes_bwd=1e10),
             mk(feat_bytes_local=1e8, hidden_bytes_fwd=5e9, hidden_bytes_bwd=5e9),
             mk(feat_bytes_local=1e8, hidden_bytes_fwd=2e9, hidden_bytes_bwd=2e9)]
    alpha = [1e-5] * 8
    beta = [1e12] * 8
    tb = [[0.0]] * 4
    pred, pick = S.predict(stats, alpha, beta, tb)
    assert pick == 0 and pred[0] == pytest.approx(2e9 / 1e12 + 2e-5)
    beta2 = list(beta)
    beta2[S.OP_PEER_PULL] = 1e9                                # slow peer reads -> DNP
    pred2, pick2 = S.predict(stats, alpha, beta2, tb)
    assert pick2 == 3 and pred2[3] < pred2[2] < pred2[1]


def test_tiered_store_classification_invariants(tiny_graph):
    """Tiers of the unified store: with everything in HBM and no cache the
    classification is the plain partition one; the host tier holds exactly the rows past
    each partition's HBM budget; a cached row is local for its rank only."""
    C, n = 4, tiny_graph.n
    part = aptgen.partition(n, C)
    ids = np.arange(n)
    plain = S.tiered_store(part, C, 1.0)
    for r in range(C):
        assert np.array_equal(plain(r, ids), np.where(part == r, 0, 1))
    t = S.tiered_store(part, C, 0.25)
    n_host = sum(len(np.nonzero(part == o)[0]) - int(np.ceil(0.25 * (part == o).sum())) for o in range(C))
    assert (t(0, ids) == 2).sum() == n_host
    hot = np.arange(0, n, 97)[:50]                          # spread over all partitions
    tc = S.tiered_store(part, C, 0.25, hot, 50)
    for r in range(C):
        newly_local = (tc(r, ids) == 0) & (t(r, ids) != 0)
        # every candidate not already in r's HBM is replicated on r, nothing else changes
        assert newly_local.sum() == int((t(r, hot) != 0).sum()) > 0
        assert np.all(np.isin(ids[newly_local], hot))
        assert np.array_equal(tc(r, ids)[~newly_local], t(r, ids)[~newly_local])


@pytest.mark.parametrize("C", [2, 4])
def test_predict_prices_each_term_with_its_operator(tiny_graph, tiny_cfg, C):
    """Eq. 2 branch by branch.  (1) alpha = 0, T_build = 0 and a DIFFERENT beta
    for every operator: each strategy's prediction is exactly its own byte terms, each over
    its own operator -- feature rows local / peer; NFP's graph all-gather,
    forward reduce-scatter and backward all-gather (Z15); SNP / DNP's all-to-alls (Z16)
    -- maximised over ranks (Z13).  (2) beta -> infinity, a DIFFERENT alpha per operator:
    exactly its calls x alpha (Z23).  (3) the hidden bytes priced are the paper's volumes
    (P:147 NFP 2d'CN_d of which (C-1)/C crosses the wire, P:148 SNP 2d'N_vs, P:161 DNP
    2d'N_vd), written out here from N_d, N_vs, N_vd.  A mis-assigned beta or alpha fails."""
    d, dd, hb = tiny_cfg.dim, tiny_cfg.hidden, 4
    beta = [1.0e9 * (i + 2) for i in range(8)]            # all distinct
    alpha = [1.0e-6 * (i + 3) for i in range(8)]
    stats, exp_b, exp_a = [], [], []
    for s in S.STRATEGIES:
        blocks, part, gb, seeds = _rank_blocks(tiny_graph, tiny_cfg, C, s)
        st = S.emulate_layer1(s, blocks, part, C, d, dd)
        for x in st:
            x["steps"] = 1
        stats.append(st)
        tb, ta = [], []
        for x in st:
            t = x["feat_bytes_local"] / beta[S.OP_LOCAL_GATHER] + x["feat_bytes_peer"] / beta[S.OP_PEER_PULL]
            a = alpha[S.OP_LOCAL_GATHER] + (alpha[S.OP_PEER_PULL] if x["feat_bytes_peer"] else 0.0)
            if s == "NFP":
                t += (x["graph_bytes"] + x["hidden_bytes_bwd"]) / beta[S.OP_ALLGATHER] \
                    + x["hidden_bytes_fwd"] / beta[S.OP_REDUCE_SCATTER]
                a += 2 * alpha[S.OP_ALLGATHER] + alpha[S.OP_REDUCE_SCATTER]
            elif s in ("SNP", "DNP"):
                t += (x["graph_bytes"] + x["hidden_bytes_fwd"] + x["hidden_bytes_bwd"]) / beta[S.OP_ALLTOALLV]
                a += 3 * alpha[S.OP_ALLTOALLV]
            tb.append(t)
            ta.append(a)
        exp_b.append(max(tb))
        exp_a.append(max(ta))
        hidden = sum(x["hidden_bytes_fwd"] + x["hidden_bytes_bwd"] for x in st)
        if s == "NFP":
            assert hidden * C == 2 * dd * C * sum(x["n_d"] for x in st) * hb * (C - 1)
        elif s == "SNP":
            assert hidden == 2 * dd * sum(x["n_vs"] for x in st) * hb
        elif s == "DNP":
            assert hidden == 2 * dd * sum(x["n_vd"] for x in st) * hb
        else:
            assert hidden == 0
    zero = [[0.0] * C for _ in range(4)]
    pred, pick = S.predict(stats, [0.0] * 8, beta, zero)
    assert pred == pytest.approx(exp_b, rel=1e-12) and pick == int(np.argmin(exp_b))
    pred_a, _ = S.predict(stats, alpha, [1e300] * 8, zero)
    assert pred_a == pytest.approx(exp_a, rel=1e-12)


def test_epoch_perm_is_sorted_by_philox_key_then_id():
    """O1 exactly: perm = train ascending by (key, u), key(u) = word0 | word1 << 32 of
    Philox_PERM(seed; {u_lo, u_hi, epoch, 0}) -- keys recomputed here from the KAT-pinned
    Philox block function (oracle.philox), not from orc_perm_key.  Ties (none expected
    among 64-bit keys) break by u; checked on the full order."""
    train = np.arange(7, 40000, 5, dtype=np.int64)
    seed, epoch = 0x1234_5678_9ABC, 3
    perm = oracle.epoch_perm(train, seed, epoch)
    key = (seed & 0xFFFFFFFF, ((seed >> 32) & 0xFFFFFFFF) ^ oracle.DOMAIN["PERM"])
    keys = {}
    for u in train:
        w = oracle.philox([u & 0xFFFFFFFF, u >> 32, epoch, 0], key)
        keys[int(u)] = int(w[0]) | (int(w[1]) << 32)
    expect = sorted(train.tolist(), key=lambda u: (keys[u], u))
    assert perm.tolist() == expect


@pytest.mark.parametrize("strategy", ["GDP", "NFP", "SNP", "DNP"])
def test_cache_sets_follow_p163(tiny_graph, tiny_cfg, strategy):
    """P:163's cache rules, checked by brute force against their text: every cached node
    is a candidate of the rule (SNP: own partition; DNP: partition + 1-hop neighbours;
    GDP/NFP: any node), the set has min(budget, #candidates) nodes, and no uncached
    candidate is more popular than a cached one (ties: the smaller id is cached)."""
    g, C, budget = tiny_graph, 4, 700
    part = aptgen.partition(g.n, C)
    counts = S.access_counts(g, aptgen.train_nodes(g, tiny_cfg), tiny_cfg.fanouts, tiny_cfg.sample_seed, 0, C,
                             tiny_cfg.batch, 2)
    sets = S.cache_sets(strategy, counts, part, C, budget, g.indptr, g.indices)
    for r in range(C):
        if strategy in ("GDP", "NFP"):
            cand = set(range(g.n))
        elif strategy == "SNP":
            cand = {u for u in range(g.n) if part[u] == r}
        else:
            own = [u for u in range(g.n) if part[u] == r]
            cand = set(own) | {int(v) for u in own for v in g.indices[g.indptr[u]:g.indptr[u + 1]]}
        got = [int(u) for u in sets[r]]
        assert len(got) == len(set(got)) == min(budget, len(cand))
        assert set(got) <= cand
        rest = cand - set(got)
        key = lambda u: (-int(counts[u]), u)
        if rest:
            assert max(key(u) for u in got) < min(key(u) for u in rest)
        assert got == sorted(got, key=key)                 # hottest first
    if strategy in ("GDP", "NFP"):
        assert all(np.array_equal(sets[0], x) for x in sets)


def test_cached_store_feature_map():
    """own cache first, else a peer GPU's cache (NVLink), else the host."""
    sets = [np.array([0, 1]), np.array([1, 2]), np.array([], np.int64)]
    tier = S.cached_store(sets, 5)
    assert tier(0, [0, 1, 2, 3]).tolist() == [0, 0, 1, 2]
    assert tier(1, [0, 1, 2, 4]).tolist() == [1, 0, 0, 2]
    assert tier(2, [0, 1, 2, 3]).tolist() == [1, 1, 1, 2]
