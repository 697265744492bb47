"""Parity of the exact benchmarked configuration (-m gpu).

BASELINE.json configs[1] as bench.py times it: synthetic ogbn-products shape (R-MAT 2.4 M
nodes / 62 M edges), 3-layer GraphSAGE 100 -> 256 -> 256 -> 47 ("3 layers"), fanout
[10, 10, 10], B = 1024, GDP at C = 1, CUDA-graph replay with the next step's sampling
pipelined, SGD update inside the step -- compared element by element with the fp64 oracle
(oracle/model.py) on the same seeds: every layer's Z and H, the logits, the loss, every
dW / db, and the parameters after the SGD update.  Both dtypes (f32, bf16); bf16 also
against the UNROUNDED fp64 definition (north star: bf16 paths within 2e-2 relative).
Tolerances: tests/parity_util.py.
"""
import numpy as np
import pytest

import aptgen
import oracle
from oracle import model
from parity_util import assert_close, reconcile

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

LR = 0.05   # bench.py make_trainer


@pytest.fixture(scope="module")
def products():
    cfg = aptgen.CONFIGS["products"]
    g = aptgen.make_graph(cfg)
    return cfg, g, aptgen.train_nodes(g, cfg), aptgen.labels(cfg, g.n)


@pytest.fixture(scope="module")
def A():
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    A.lib()
    return A


def _bench_trainer(A, cfg, g, train, labels, dtype):
    """The trainer exactly as bench.py builds it (stream, graph replay, pipelining)."""
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(priority=-1)
    ctx = A.Ctx(0, 1, 0, stream.cuda_stream)
    gr = ctx.graph_load(g.indptr, g.indices)
    dt = A.DTYPE[dtype]
    fs = ctx.fstore_create(gr, A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, LR, cfg.sample_seed, cfg.feat_seed, A.GDP, labels)
    tr.set_params(aptgen.weights(cfg))
    tr.set_epoch(train, 0)
    tr.use_graph(True)
    return ctx, tr


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_products_bench_step_matches_oracle(A, products, dtype):
    cfg, g, train, labels = products
    ctx, tr = _bench_trainer(A, cfg, g, train, labels, dtype)
    for s in range(2):                                   # warm-up steps with the update, as the bench
        tr.step(s, update=True)
    p_before = tr.get_params()
    step = 2
    tr.step(step, update=True)                           # the timed graph variant: pipelined, update = 1
    p_after = tr.get_params()
    seeds = tr.read("seeds")[:, 0].astype(np.int64)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    assert np.array_equal(seeds, perm[step * cfg.batch:(step + 1) * cfg.batch])
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, step)
    K = len(blocks)
    assert K == 3
    for l in range(1, K + 1):
        assert np.array_equal(tr.read("dst", l)[:, 0], blocks[K - l].dst), f"layer {l} dst"
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in p_before]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), dtype, lr=LR)
    # layer-1 Z is bit-exact under O4 (exact sums, IEEE division; bf16 mode: then RNE to bf16)
    assert np.array_equal(tr.read("Z", 1), ref["cache"]["Z"][0].astype(np.float32))
    ref, bd = reconcile(blocks, p64, ref, dtype, len(seeds), [tr.read("H", l) for l in range(1, K)])
    for l in range(1, K + 1):
        assert_close(tr.read("H", l), ref["cache"]["h"][l - 1], dtype, f"H layer {l}", bd["H"][l - 1])
    loss = tr.loss()
    assert abs(loss - ref["loss"]) <= (1e-5 if dtype == "f32" else 2e-2) * abs(ref["loss"]), (loss, ref["loss"])
    for l in range(1, K + 1):
        dW, db = ref["grads"][l - 1]
        assert_close(tr.read("dW", l), dW, dtype, f"dW layer {l}", bd["dW"][l - 1])
        assert_close(tr.read("db", l)[0], db, dtype, f"db layer {l}", bd["db"][l - 1])
    # the SGD update inside the step: W' = W - lr dW (fp32 master weights)
    for l, ((Wa, ba), (Wb, bb), (dW, db)) in enumerate(zip(p_after, p_before, ref["grads"]), start=1):
        got_dW = (Wb.astype(np.float64) - Wa) / LR
        got_db = (bb.astype(np.float64) - ba) / LR
        # the fp32 subtraction rounds W' to half an ulp of |W|: that, / lr, is the floor
        fl_W = np.abs(Wb).astype(np.float64) * 2.0 ** -23 / LR
        fl_b = np.abs(bb).astype(np.float64) * 2.0 ** -23 / LR
        assert_close(got_dW, dW, dtype, f"SGD W layer {l}", bd["dW"][l - 1] + fl_W)
        assert_close(got_db, db, dtype, f"SGD b layer {l}", bd["db"][l - 1] + fl_b)
    tr.close()
    ctx.close()


def test_products_bench_step_bf16_vs_unrounded_fp64(A, products):
    """The bf16 path (features, Z, W, hidden activations and the backward operands rounded
    to bf16) against the fp64 definition with NO rounding points emulated: every layer's H,
    the loss and every dW / db within the north star's bf16 bar (2e-2 relative; reading T2)."""
    cfg, g, train, labels = products
    ctx, tr = _bench_trainer(A, cfg, g, train, labels, "bf16")
    tr.step(0, update=False)
    step = 1
    tr.step(step, update=False)
    seeds = tr.read("seeds")[:, 0].astype(np.int64)
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, step)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in aptgen.weights(cfg)]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), "f32")
    K = len(blocks)
    ref, bd = reconcile(blocks, p64, ref, "bf16u", len(seeds), [tr.read("H", l) for l in range(1, K)])
    for l in range(1, K + 1):
        assert_close(tr.read("H", l), ref["cache"]["h"][l - 1], "bf16u", f"H layer {l} (unrounded ref)", bd["H"][l - 1])
    assert abs(tr.loss() - ref["loss"]) <= 2e-2 * abs(ref["loss"])
    for l in range(1, K + 1):
        dW, db = ref["grads"][l - 1]
        assert_close(tr.read("dW", l), dW, "bf16u", f"dW layer {l} (unrounded ref)", bd["dW"][l - 1])
        assert_close(tr.read("db", l)[0], db, "bf16u", f"db layer {l} (unrounded ref)", bd["db"][l - 1])
    tr.close()
    ctx.close()


def test_products_epoch_permutation_full_train(A, products):
    """S1 at full size: the device permutation (Philox keys + the library's radix sort) of a
    1.2 M-id train set equals oracle.epoch_perm, read back through the seeds of the first,
    a middle and the short last step (O1, R6)."""
    cfg, g, _, labels = products
    train = np.arange(1, g.n, 2, dtype=np.int64)           # 1.2 M ascending ids
    ctx, tr = _bench_trainer(A, cfg, g, train, labels, "bf16")
    tr.set_epoch(train, 5)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 5)
    spe = tr.steps_per_epoch()
    assert spe == -(-len(train) // cfg.batch)
    for s in (0, spe // 2, spe - 1):
        tr.step(s, update=False)
        assert np.array_equal(tr.read("seeds")[:, 0], perm[s * cfg.batch:(s + 1) * cfg.batch]), s
    tr.close()
    ctx.close()


@pytest.mark.parametrize("strategy,C", [("NFP", 2), ("SNP", 2), ("DNP", 2), ("SNP", 4), ("DNP", 4), ("GDP", 4)])
def test_products_strategies_match_oracle(A, products, strategy, C):
    """Every strategy at the benchmark's scale (products shape, 3 layers, B = 1024 per rank,
    bf16, CUDA graph + pipelined sampling) with C ranks emulated on this B200: every rank's
    every-layer H, the loss and every all-reduced dW / db against the oracle's per-rank fp64
    model (the strategies compute the same function), within the derived
    bounds (T1-T3)."""
    from oracle import strategy as S
    from parity_util import sum_bounds
    cfg, g, train, labels = products
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(priority=-1)
    ctx = A.Ctx(-1, C, 0, stream.cuda_stream)
    part = aptgen.partition(g.n, C)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, A.BF16, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.BF16, LR, cfg.sample_seed, cfg.feat_seed,
                   A.STRATEGY[strategy], labels)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    tr.set_epoch(train, 0)
    tr.use_graph(True)
    tr.step(0, update=False)
    step = 1
    tr.step(step, update=False)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, step, C, cfg.batch)
    seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
    K = len(cfg.fanouts)
    refs, bds = [], []
    for r in range(C):
        assert np.array_equal(tr.read("seeds", rank=r)[:, 0], seeds[r])
        blocks = oracle.sample_blocks(g, seeds[r], cfg.fanouts, cfg.sample_seed, step)
        ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds[r]], len(gb), "bf16",
                               snp=(part, C) if strategy == "SNP" else None)
        ref, bd = reconcile(blocks, p64, ref, "bf16", len(gb), [tr.read("H", l, rank=r) for l in range(1, K)])
        refs.append(ref)
        bds.append(bd)
        for l in range(1, K + 1):
            assert_close(tr.read("H", l, rank=r), ref["cache"]["h"][l - 1], "bf16", f"H{l} rank {r}", bd["H"][l - 1])
    loss = sum(x["loss"] for x in refs)
    assert abs(tr.loss() - loss) <= 2e-2 * abs(loss)
    sb = sum_bounds(bds)
    for l in range(1, K + 1):
        for r in (0, C - 1):
            assert_close(tr.read("dW", l, rank=r), sum(x["grads"][l - 1][0] for x in refs), "bf16",
                         f"dW{l} rank {r}", sb["dW"][l - 1])
            assert_close(tr.read("db", l, rank=r)[0], sum(x["grads"][l - 1][1] for x in refs), "bf16",
                         f"db{l} rank {r}", sb["db"][l - 1])
    tr.close()
    ctx.close()
