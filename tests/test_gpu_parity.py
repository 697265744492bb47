"""GPU parity: the sm_100a path through the C ABI vs the CPU oracle (-m gpu).

Bars (BASELINE.json north_star): sampled blocks and indices bit-exact; Z under the
O4 features bit-exact; fp32 outputs and gradients rtol 1e-5 / atol 1e-6; bf16
paths rtol 2e-2 (atol derived in DESIGN.md §Tolerances).
"""
import numpy as np
import pytest

import aptgen
import oracle
from oracle import model
from parity_util import assert_close, reconcile, sum_bounds, t1

pytestmark = pytest.mark.gpu
LAMBDA_U = 6 * 2.0 ** -24       # one fp32 rounding of the bias add, at LAMBDA

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def A():
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    A.lib()
    return A


@pytest.fixture(scope="module")
def ctx(A):
    torch.cuda.set_device(0)
    return A.Ctx(0, 1, 0)


@pytest.fixture(scope="module")
def tiny(tiny_cfg, tiny_graph):
    return tiny_cfg, tiny_graph, aptgen.train_nodes(tiny_graph, tiny_cfg)


def dev_i64(a):
    return torch.as_tensor(np.ascontiguousarray(a, np.int64)).cuda()


# ------------------------------------------------------------------ S2 / S3
@pytest.mark.parametrize("step", [0, 1, 5])
def test_sample_blocks_bit_exact_tiny(A, ctx, tiny, step):
    cfg, g, train = tiny
    gr = ctx.graph_load(g.indptr, g.indices)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    seeds = perm[step * cfg.batch:(step + 1) * cfg.batch]
    sd = dev_i64(seeds)
    b = ctx.sample(gr, sd, len(seeds), cfg.fanouts, cfg.sample_seed, step)
    ref = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, step)
    for h, rb in enumerate(ref):
        dst, src, indptr, indices = b.block_host(h)
        assert np.array_equal(dst, rb.dst)
        assert np.array_equal(src, rb.src)
        assert np.array_equal(indptr, rb.indptr)
        assert np.array_equal(indices, rb.indices)


@pytest.mark.parametrize("fanouts", [(1, 3), (25, 7), (40,), (256, 2)])
def test_sample_edge_fanouts(A, ctx, tiny, fanouts):
    """fanout 1, > 32 (multi-slot Floyd), 256 (max) and deg <= k rows."""
    cfg, g, train = tiny
    gr = ctx.graph_load(g.indptr, g.indices)
    seeds = train[::7][:300]
    b = ctx.sample(gr, dev_i64(seeds), len(seeds), fanouts, 11, 3)
    ref = oracle.sample_blocks(g, seeds, fanouts, 11, 3)
    for h, rb in enumerate(ref):
        dst, src, indptr, indices = b.block_host(h)
        assert np.array_equal(src, rb.src) and np.array_equal(indptr, rb.indptr)
        assert np.array_equal(indices, rb.indices)


def test_sample_empty_and_isolated(A, ctx, tiny):
    cfg, g, _ = tiny
    gr = ctx.graph_load(g.indptr, g.indices)
    iso = np.nonzero(g.degrees() == 0)[0][:5].astype(np.int64)
    b = ctx.sample(gr, dev_i64(iso), len(iso), (3, 3), 1, 0)
    v = b.block(0)
    assert v.n_dst == len(iso) and v.n_edges == 0 and v.n_src == len(iso)
    b0 = ctx.sample(gr, dev_i64(np.zeros(0)), 0, (3, 3), 1, 0)
    assert b0.block(1).n_dst == 0


@pytest.mark.slow
def test_sample_products_bit_exact(A, ctx):
    cfg = aptgen.CONFIGS["products"]
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    gr = ctx.graph_load(g.indptr, g.indices)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    for step in (0, 17):
        seeds = perm[step * cfg.batch:(step + 1) * cfg.batch]
        b = ctx.sample(gr, dev_i64(seeds), len(seeds), cfg.fanouts, cfg.sample_seed, step)
        ref = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, step)
        for h, rb in enumerate(ref):
            dst, src, indptr, indices = b.block_host(h)
            assert np.array_equal(src, rb.src) and np.array_equal(indices, rb.indices)
            assert np.array_equal(indptr, rb.indptr)


# ------------------------------------------------------------------ features / gather
@pytest.mark.parametrize("dtype,dim", [("f32", 64), ("bf16", 100), ("f32", 100), ("bf16", 256)])
def test_feature_store_bit_exact(A, ctx, tiny, dtype, dim):
    cfg, g, _ = tiny
    gr = ctx.graph_load(g.indptr, g.indices)
    fs = ctx.fstore_create(gr, A.GDP, A.DTYPE[dtype], dim, None, cfg.feat_seed)
    ids = np.array([0, 1, 2, 77, 4095, 9999, 5000, 5000], np.int32)
    pitch = ((dim + 7) // 8 * 8) if dtype == "bf16" else ((dim + 3) // 4 * 4)
    esz = 2 if dtype == "bf16" else 4
    out = torch.zeros(len(ids) * pitch * esz, dtype=torch.uint8, device="cuda")
    ctx.gather(fs, torch.as_tensor(ids.astype(np.int64)).cuda(), len(ids), out)
    torch.cuda.synchronize()
    raw = out.cpu().numpy()
    if dtype == "bf16":
        got = (raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32).reshape(len(ids), pitch)[:, :dim]
    else:
        got = raw.view(np.float32).reshape(len(ids), pitch)[:, :dim]
    ref = oracle.features(cfg.feat_seed, ids.astype(np.int64), dim)
    assert np.array_equal(got.astype(np.float64), ref)


# ------------------------------------------------------------------ S7 aggregation
def test_mean_division_is_ieee_exhaustive(A, ctx):
    """The mean divides with a per-row reciprocal + one FMA correction (Markstein); it must
    agree bit for bit with IEEE x/d on every O4 mean (O5) -- 67M operands."""
    assert A.lib().apt_selftest_div() == 0

@pytest.mark.parametrize("n,bits", [(1, 64), (2049, 3), (300001, 12), (1200000, 64), (65536, 1)])
def test_epoch_sort_stable_radix(A, ctx, n, bits):
    """S1's own radix sort (sort.cu) is a STABLE sort by the 64-bit key (equal keys keep the
    input order, reading O1's tie rule): against a host stable sort, with many equal keys."""
    assert A.lib().apt_selftest_sort(n, 77, bits) == 0


def test_aggregate_bit_exact_and_bwd(A, ctx, tiny):
    cfg, g, train = tiny
    gr = ctx.graph_load(g.indptr, g.indices)
    seeds = train[:200]
    b = ctx.sample(gr, dev_i64(seeds), len(seeds), (6,), 5, 2)
    (rb,) = oracle.sample_blocks(g, seeds, (6,), 5, 2)
    d = 36
    x = oracle.features(cfg.feat_seed, rb.src, d)
    xd = torch.as_tensor(x.astype(np.float32)).cuda().contiguous()
    z = torch.zeros((rb.n_dst, 36), dtype=torch.float32, device="cuda")
    v = b.block(0)
    ctx.aggregate(v, xd, A.F32, d, d, z, 36)
    ref = oracle.aggregate(rb.indptr, rb.indices, x)
    assert np.array_equal(z.cpu().numpy(), ref.astype(np.float32))          # exact under O4
    dz = np.random.default_rng(0).normal(size=(rb.n_dst, d)).astype(np.float32)
    dx = torch.zeros((rb.n_src, d), dtype=torch.float32, device="cuda")
    ctx.aggregate_bwd(v, torch.as_tensor(dz).cuda(), d, d, dx, d)
    refb = oracle.aggregate_bwd(rb.indptr, rb.indices, dz.astype(np.float64), rb.n_src)
    assert np.allclose(dx.cpu().numpy(), refb, rtol=1e-5, atol=1e-6)


# ------------------------------------------------------------------ S8 projection
@pytest.mark.parametrize("M,N,K", [(1, 16, 64), (127, 32, 64), (128, 47, 100), (1000, 256, 100),
                                   (5000, 256, 256), (333, 48, 256), (4099, 8, 16), (1000, 512, 384),
                                   (300, 1040, 64)])
def test_project_tcgen05_bf16(A, ctx, M, N, K):
    rng = np.random.default_rng(M + N + K)
    kp = (K + 7) // 8 * 8
    Z = oracle.bf16_round(rng.normal(size=(M, K)))
    W = (rng.normal(size=(N, K)) / np.sqrt(K)).astype(np.float32)
    bias = rng.normal(size=N).astype(np.float32)
    Zb = np.zeros((M, kp), np.uint16)
    Zb[:, :K] = (Z.astype(np.float32).view(np.uint32) >> 16).astype(np.uint16)
    yp = (N + 3) // 4 * 4
    Y = torch.zeros((M, yp), dtype=torch.float32, device="cuda")
    ctx.project(torch.as_tensor(Zb.view(np.int16)).cuda(), kp, A.BF16, torch.as_tensor(W).cuda(),
                torch.as_tensor(bias).cuda(), M, N, K, 1, Y, yp)
    Wr = oracle.bf16_round(W)
    ref = np.maximum(Z @ Wr.T + bias, 0)
    got = Y.cpu().numpy()[:, :N]
    # fp32 accumulation of bf16 products: the fp32 bar with the T1 allowance
    assert_close(got, ref, "f32", "Y", t1(np.abs(Z), np.abs(Wr).T, K) + LAMBDA_U * np.abs(bias))


@pytest.mark.parametrize("f32", [1, 0])
@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 0), (1, 1)])
@pytest.mark.parametrize("M,N,K,acc", [(64, 32, 32, 0), (64, 32, 64, 1), (300, 70, 100, 0), (130, 300, 1000, 1),
                                       (1, 8, 8, 0), (4099, 264, 72, 1)])
def test_general_tensor_core_gemm(A, ctx, f32, a_mn, b_mn, M, N, K, acc):
    """The general tcgen05 contraction (gemm_tc_gen.cu) in every operand layout: fp32 as
    3xTF32 (each product carried to ~2^-21 of its magnitude: reading P1), bf16 exact
    operands with fp32 accumulation; N tiled past 256, K streamed, split-K accumulating.
    Error relative to sum_k |A||B| + |b| (the T1 scale of the sum)."""
    err = A.lib().apt_selftest_gemm(f32, a_mn, b_mn, M, N, K, acc)
    assert 0 <= err < (2e-6 if f32 else 5e-7), err


@pytest.mark.parametrize("M,N,K", [(1, 5, 3), (1, 8, 4), (130, 47, 100), (2000, 256, 100), (49537, 256, 100),
                                   (3001, 300, 520), (700, 1024, 256), (257, 40, 1030)])
def test_project_fp32(A, ctx, M, N, K):
    """fp32 mode on the tensor cores (3xTF32, kind::tf32; K = 3 / N = 5 fall back to CUDA
    cores: pitches not 16-byte multiples), N tiled past 256 and K streamed past 256."""
    rng = np.random.default_rng(7)
    Z = rng.normal(size=(M, K)).astype(np.float32)
    W = rng.normal(size=(N, K)).astype(np.float32)
    bias = rng.normal(size=N).astype(np.float32)
    Y = torch.zeros((M, N), dtype=torch.float32, device="cuda")
    ctx.project(torch.as_tensor(Z).cuda(), K, A.F32, torch.as_tensor(W).cuda(), torch.as_tensor(bias).cuda(),
                M, N, K, 0, Y, N)
    ref = Z.astype(np.float64) @ W.T.astype(np.float64) + bias
    assert_close(Y.cpu().numpy(), ref, "f32", "Y", t1(np.abs(Z), np.abs(W).T, K) + LAMBDA_U * np.abs(bias))


# ------------------------------------------------------------------ the training step (C = 1)
def _trainer(A, ctx, cfg, g, train, dtype, strategy="GDP", lr=0.1):
    gr = ctx.graph_load(g.indptr, g.indices)
    fs = ctx.fstore_create(gr, A.STRATEGY[strategy] if strategy == "NFP" else A.GDP, A.DTYPE[dtype], cfg.dim, None,
                           cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    labels = aptgen.labels(cfg, g.n)
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.DTYPE[dtype], lr, cfg.sample_seed, cfg.feat_seed,
                   A.STRATEGY[strategy], labels)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    tr.set_epoch(train, 0)
    return tr, params, labels




def _check_grads(tr, ref, bd, dtype, K, rank=0, what=""):
    for l in range(1, K + 1):
        dW, db = ref["grads"][l - 1]
        assert_close(tr.read("dW", l, rank=rank), dW, dtype, f"{what}dW layer {l}", bd["dW"][l - 1])
        assert_close(tr.read("db", l, rank=rank)[0], db, dtype, f"{what}db layer {l}", bd["db"][l - 1])


# fanouts: tiny's [5,5]; 3 layers like the benchmarked model; layer-1 fanouts 16 and
# 12 (the two-nodes-per-warp sampler at its k = 16 limit, the layer-1 gather's 5-load rounds
# with a ragged last round, k in 11..16)
FANOUTS = [(5, 5), (5, 5, 5), (16, 12), (12, 16)]


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("step", [0, 3])
@pytest.mark.parametrize("fanouts", FANOUTS)
def test_train_step_matches_oracle(A, ctx, tiny, dtype, step, fanouts):
    cfg, g, train = tiny
    cfg = cfg.replace(fanouts=fanouts)
    tr, params, labels = _trainer(A, ctx, cfg, g, train, dtype)
    tr.step(step, update=False)
    loss = tr.loss()
    seeds = tr.read("seeds")[:, 0].astype(np.int64)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    assert np.array_equal(seeds, perm[step * cfg.batch:(step + 1) * cfg.batch])
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, step)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), dtype)
    K = len(blocks)
    for l in range(1, K + 1):
        assert np.array_equal(tr.read("dst", l)[:, 0], blocks[K - l].dst)
    # layer-1 Z is bit-exact under O4 features (exact sums, IEEE division)
    assert np.array_equal(tr.read("Z", 1), ref["cache"]["Z"][0].astype(np.float32))
    ref, bd = reconcile(blocks, p64, ref, dtype, len(seeds), [tr.read("H", l) for l in range(1, K)])
    for l in range(1, K + 1):
        assert_close(tr.read("H", l), ref["cache"]["h"][l - 1], dtype, f"H layer {l}", bd["H"][l - 1])
    assert abs(loss - ref["loss"]) <= (1e-5 if dtype == "f32" else 2e-2) * abs(ref["loss"])
    _check_grads(tr, ref, bd, dtype, K)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_train_step_wide_hidden(A, ctx, tiny, dtype):
    """Hidden width past every single-launch limit (config 5 sweeps d' to 1024): the upper
    layer's aggregation and the pull backward run in 512-column chunks, the projections
    and weight gradients on the CUDA-core fallback (bf16 mode reads the bf16 gradient)."""
    cfg, g, train = tiny
    cfg = cfg.replace(hidden=1040)
    tr, params, labels = _trainer(A, ctx, cfg, g, train, dtype)
    tr.step(1, update=False)
    seeds = tr.read("seeds")[:, 0].astype(np.int64)
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, 1)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), dtype)
    K = len(blocks)
    ref, bd = reconcile(blocks, p64, ref, dtype, len(seeds), [tr.read("H", l) for l in range(1, K)])
    for l in range(1, K + 1):
        assert_close(tr.read("H", l), ref["cache"]["h"][l - 1], dtype, f"H layer {l}", bd["H"][l - 1])
    assert abs(tr.loss() - ref["loss"]) <= (1e-5 if dtype == "f32" else 2e-2) * abs(ref["loss"])
    _check_grads(tr, ref, bd, dtype, K)


@pytest.mark.parametrize("use_graph", [False, True])
def test_step_host_pipelined_matches_device_steps(A, ctx, tiny, use_graph):
    """The pipelined end-to-end call (submit batch t+1, run batch t) returns, call by call,
    the losses of the device-resident steps on the same batches."""
    cfg, g, train = tiny
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    tr, params, labels = _trainer(A, ctx, cfg, g, train, "bf16")
    tr.use_graph(use_graph)
    ref = []
    for step in range(3):
        tr.step(step, update=False)
        ref.append(tr.loss())
    tr2, _, _ = _trainer(A, ctx, cfg, g, train, "bf16")
    tr2.use_graph(use_graph)
    got = []
    for step in range(4):
        nxt = torch.as_tensor(perm[(step % 3) * cfg.batch:((step % 3) + 1) * cfg.batch]).pin_memory()
        loss = tr2.step_host_pipelined(nxt, step % 3, update=False)
        if step == 0:
            assert loss is None
        else:
            got.append(loss)
    assert np.allclose(got, ref, rtol=1e-6)


@pytest.mark.parametrize("use_graph", [False, True])
def test_step_host_async_matches_device_steps(A, ctx, tiny, use_graph):
    """The asynchronous end-to-end call returns, one call late, the losses of the
    device-resident steps on the same batches (and the last one via apt_trainer_loss)."""
    cfg, g, train = tiny
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    tr, params, labels = _trainer(A, ctx, cfg, g, train, "bf16")
    tr.use_graph(use_graph)
    ref = []
    for step in range(4):
        tr.step(step % 3, update=False)
        ref.append(tr.loss())
    tr2, _, _ = _trainer(A, ctx, cfg, g, train, "bf16")
    tr2.use_graph(use_graph)
    got = []
    for call in range(5):
        nxt = torch.as_tensor(perm[(call % 3) * cfg.batch:((call % 3) + 1) * cfg.batch]).pin_memory()
        loss = tr2.step_host_async(nxt, call % 3, update=False)
        if call < 2:
            assert loss is None
        else:
            got.append(loss)
    got.append(tr2.loss())             # the last launched step (batch 3 % 3)
    assert np.allclose(got, ref, rtol=1e-6), (got, ref)


@pytest.mark.parametrize("strategy,C", [("GDP", 1), ("SNP", 2), ("NFP", 2), ("DNP", 2)])
def test_pipelined_steps_equal_unpipelined(A, tiny, strategy, C):
    """Sampling step t+1 during step t (two sample sets, second stream) changes nothing:
    eager/graph x pipelined/unpipelined give the same parameters after 4 updates, with a
    non-sequential step id in the middle (the prefetch is discarded and redone)."""
    cfg, g, train = tiny
    outs = []
    for use_graph, pipe in ((False, False), (True, False), (False, True), (True, True)):
        ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
        gr = ctx.graph_load(g.indptr, g.indices, aptgen.partition(g.n, C))
        fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, A.F32, cfg.dim, None, cfg.feat_seed)
        dims = [cfg.dim] + [d for _, d in cfg.dims()]
        tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.F32, 0.3, cfg.sample_seed, cfg.feat_seed,
                       A.STRATEGY[strategy], aptgen.labels(cfg, g.n))
        tr.set_params(aptgen.weights(cfg))
        tr.set_epoch(train, 0)
        tr.use_graph(use_graph)
        tr.set_pipeline(pipe)
        spe = tr.steps_per_epoch()
        for s in (0, 1, 0, 1 % spe):
            tr.step(s % spe, update=True)
        outs.append((tr.get_params(), tr.read("seeds")[:, 0]))
    for params, seeds in outs[1:]:
        assert np.array_equal(seeds, outs[0][1])
        for (W0, b0), (W1, b1) in zip(outs[0][0], params):
            assert np.allclose(W0, W1, rtol=1e-5, atol=1e-6) and np.allclose(b0, b1, rtol=1e-5, atol=1e-6)


def test_sgd_update_and_graph_replay(A, ctx, tiny):
    """Two steps with the update, eager vs CUDA-graph replay: identical parameters."""
    cfg, g, train = tiny
    outs = []
    for use_graph in (False, True):
        tr, params, labels = _trainer(A, ctx, cfg, g, train, "f32", lr=0.5)
        tr.use_graph(use_graph)
        for s in range(3):
            tr.step(s, update=True)
        outs.append(tr.get_params())
    for (W0, b0), (W1, b1) in zip(*outs):
        assert np.allclose(W0, W1, rtol=1e-6, atol=1e-7), np.abs(W0 - W1).max()
        assert np.allclose(b0, b1, rtol=1e-6, atol=1e-7), np.abs(b0 - b1).max()
    # one step against the oracle's SGD
    tr, params, labels = _trainer(A, ctx, cfg, g, train, "f32", lr=0.5)
    tr.step(0, update=True)
    seeds = tr.read("seeds")[:, 0].astype(np.int64)
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, 0)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), "f32", lr=0.5)
    for (W, b), (Wr, br) in zip(tr.get_params(), ref["new_params"]):
        assert np.allclose(W, Wr, rtol=1e-5, atol=1e-6) and np.allclose(b, br, rtol=1e-5, atol=1e-6)


@pytest.mark.parametrize("use_graph", [False, True])
def test_step_host_e2e_matches_device_step(A, ctx, tiny, use_graph):
    """The end-to-end call (host global batch in, loss out; H2D -> step -> D2H replayed as
    one graph) reproduces the device-resident step on the same seeds."""
    cfg, g, train = tiny
    tr, params, labels = _trainer(A, ctx, cfg, g, train, "bf16")
    tr.use_graph(use_graph)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    for step in (2, 1, 2):
        tr.step(step, update=False)
        l_dev = tr.loss()
        gb = torch.as_tensor(perm[step * cfg.batch:(step + 1) * cfg.batch]).pin_memory()
        l_host = tr.step_host(gb, step, update=False)
        assert l_host == pytest.approx(l_dev, rel=1e-6)
        assert np.array_equal(tr.read("seeds")[:, 0], perm[step * cfg.batch:(step + 1) * cfg.batch])


# ------------------------------------------------------------------ S11 weight gradient
@pytest.mark.parametrize("rows,d_out,d_in", [(1, 16, 64), (63, 47, 256), (64, 256, 100), (1000, 256, 256),
                                             (49537, 256, 100), (5000, 32, 64), (300, 200, 8), (2000, 1040, 256),
                                             (777, 300, 1024)])
@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_weight_grad(A, ctx, rows, d_out, d_in, dtype):
    """dW = G^T Z, db = colsum(G): tcgen05 (MN-major operands, all-ones bias column) in bf16
    mode, exact CUDA-core fp32 otherwise; against an fp64 product of the same rounded inputs."""
    rng = np.random.default_rng(rows + d_out + d_in)
    G = rng.normal(size=(rows, d_out)).astype(np.float32)
    Z = rng.normal(size=(rows, d_in))
    gp = (d_out + 3) // 4 * 4
    Gd = np.zeros((rows, gp), np.float32)
    Gd[:, :d_out] = G
    if dtype == "bf16":
        Zr = oracle.bf16_round(Z)
        zp = (d_in + 7) // 8 * 8
        Zh = np.zeros((rows, zp), np.uint16)
        Zh[:, :d_in] = (Zr.astype(np.float32).view(np.uint32) >> 16).astype(np.uint16)
        Zt = torch.as_tensor(Zh.view(np.int16)).cuda()
        Gr = oracle.bf16_round(G)
    else:
        Zr = Z.astype(np.float32).astype(np.float64)
        zp = (d_in + 3) // 4 * 4
        Zf = np.zeros((rows, zp), np.float32)
        Zf[:, :d_in] = Zr
        Zt = torch.as_tensor(Zf).cuda()
        Gr = G.astype(np.float64)
    dW = torch.zeros((d_out, d_in), dtype=torch.float32, device="cuda")
    db = torch.zeros(d_out, dtype=torch.float32, device="cuda")
    ctx.weight_grad(torch.as_tensor(Gd).cuda(), gp, Zt, zp, A.DTYPE[dtype], rows, d_out, d_in, dW, db)
    # fp32 accumulation over `rows` products of the (emulated) operands: the fp32 bar with T1
    assert_close(dW.cpu().numpy(), Gr.T @ Zr, "f32", "dW", t1(np.abs(Gr).T, np.abs(Zr), rows))
    assert_close(db.cpu().numpy(), Gr.sum(0), "f32", "db", t1(np.abs(Gr).T, np.ones(rows), rows))


# ------------------------------------------------------------------ strategies (C ranks emulated on one B200)
def _strategy_ref(cfg, g, train, labels, params, strategy, C, step, dtype, bounds=None):
    """Oracle: every rank's own blocks through the fp64 model, loss over the global batch (Z20);
    the strategies must reproduce it (P:59, P:279 'semantically equivalent')."""
    from oracle import strategy as S
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, step, C, cfg.batch)
    part = aptgen.partition(g.n, C)
    seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
    refs, bds = [], []
    for r in range(C):
        blocks = oracle.sample_blocks(g, seeds[r], cfg.fanouts, cfg.sample_seed, step)
        snp = (part, C) if strategy == "SNP" else None     # SNP's own rounding points (partials)
        refs.append(model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds[r]], len(gb), dtype, snp=snp))
        if bounds is not None:     # bounds = the trainer: reconcile with rank r's mask bits (T3)
            refs[-1], bd = reconcile(blocks, p64, refs[-1], dtype, len(gb),
                                     [bounds.read("H", l, rank=r) for l in range(1, len(cfg.fanouts))])
            bds.append(bd)
    return (seeds, refs, bds) if bounds is not None else (seeds, refs)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("C,fanouts", [(2, (5, 5)), (4, (5, 5)), (8, (5, 5)), (2, (5, 5, 5)), (4, (5, 5, 5))])
@pytest.mark.parametrize("strategy", ["GDP", "NFP", "SNP", "DNP"])
def test_strategy_step_matches_oracle(A, tiny, strategy, C, fanouts, dtype):
    cfg, g, train = tiny
    cfg = cfg.replace(fanouts=fanouts)
    ctx = A.Ctx(-1, C, 0)                      # all C ranks on this device
    gr = ctx.graph_load(g.indptr, g.indices, aptgen.partition(g.n, C))
    dt = A.DTYPE[dtype]
    fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    labels = aptgen.labels(cfg, g.n)
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, 0.1, cfg.sample_seed, cfg.feat_seed,
                   A.STRATEGY[strategy], labels)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    tr.set_epoch(train, 0)
    tr.step(0, update=False)
    seeds, refs, bds = _strategy_ref(cfg, g, train, labels, params, strategy, C, 0, dtype, bounds=tr)
    K = len(cfg.fanouts)
    for r in range(C):
        assert np.array_equal(tr.read("seeds", rank=r)[:, 0], seeds[r])
        for l in range(1, K + 1):
            assert_close(tr.read("H", l, rank=r), refs[r]["cache"]["h"][l - 1], dtype, f"H layer {l} rank {r}",
                         bds[r]["H"][l - 1])
    loss = tr.loss()
    ref_loss = sum(x["loss"] for x in refs)
    assert abs(loss - ref_loss) <= (1e-5 if dtype == "f32" else 2e-2) * abs(ref_loss)
    for l in range(1, K + 1):
        dW = sum(x["grads"][l - 1][0] for x in refs)
        db = sum(x["grads"][l - 1][1] for x in refs)
        sb = sum_bounds(bds)
        for r in (0, C - 1):
            assert_close(tr.read("dW", l, rank=r), dW, dtype, f"dW layer {l} rank {r}", sb["dW"][l - 1])
            assert_close(tr.read("db", l, rank=r)[0], db, dtype, f"db layer {l} rank {r}", sb["db"][l - 1])


# ------------------------------------------------------------------ S12/S13 planner
FIELDS = ("n_d", "rows_local", "rows_peer", "rows_host", "feat_bytes_local", "feat_bytes_peer", "feat_bytes_host",
          "graph_bytes", "hidden_bytes_fwd", "hidden_bytes_bwd", "n_calls")


@pytest.mark.parametrize("C,frac,n_hot,heads", [(2, 1.0, 0, 0), (4, 1.0, 0, 0), (4, 0.4, 300, 0), (2, 1.0, 0, 4),
                                                (4, 1.0, 0, 4)])
def test_dryrun_counts_match_oracle_and_pick(A, tiny, C, frac, n_hot, heads):
    """apt_dryrun's per-strategy, per-rank counts are integers: bit-exact against
    the oracle's emulation of every rank's blocks (O7); apt_select_strategy = oracle Eq. 2 (O8)."""
    from oracle import strategy as S
    cfg, g, train = tiny
    ctx = A.Ctx(-1, C, 0)
    part = aptgen.partition(g.n, C)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    hot = np.random.default_rng(5).choice(g.n, size=n_hot, replace=False) if n_hot else None
    fs = ctx.fstore_create(gr, A.GDP, A.F32, cfg.dim, None, cfg.feat_seed, hbm_frac=frac, hot_ids=hot)
    tier = S.tiered_store(part, C, frac, hot, n_hot) if (frac < 1.0 or n_hot) else None
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    labels = aptgen.labels(cfg, g.n)
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.F32, 0.1, cfg.sample_seed, cfg.feat_seed, A.GDP,
                   labels, gat_heads=heads)
    tr.set_epoch(train, 0)
    st = tr.dryrun(2)
    assert st.gat_heads == heads
    steps = st.steps
    assert steps == min(2, tr.steps_per_epoch())
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    ref = []
    for si, s in enumerate(S.STRATEGIES):
        tot = [dict.fromkeys(FIELDS + ("n_vs", "n_vd", "attn_bytes", "attn_feat_bytes"), 0) for _ in range(C)]
        for step in range(steps):
            gb = oracle.global_batch(perm, step, C, cfg.batch)
            seeds = S.assign_seeds(s, gb, part, C, cfg.batch)
            blocks = [oracle.sample_blocks(g, sd, cfg.fanouts, cfg.sample_seed, step)[-1] for sd in seeds]
            for r, e in enumerate(S.emulate_layer1(s, blocks, part, C, cfg.dim, cfg.hidden, 4, 4, tier=tier,
                                                   heads=heads)):
                for k in tot[r]:
                    tot[r][k] += e[k]
        for r in range(C):
            for k in FIELDS + ("attn_bytes", "attn_feat_bytes"):
                assert getattr(st, k)[si][r] == tot[r][k], (s, r, k, getattr(st, k)[si][r], tot[r][k])
            if s == "SNP":
                assert st.n_vs[r] == tot[r]["n_vs"]
            if s == "DNP":
                assert st.n_vd[r] == tot[r]["n_vd"]
        for r in range(C):
            tot[r]["steps"] = steps
        ref.append(tot)
    bw = ctx.profile_links()
    assert bw.beta_Bps[0] > 1e11 and bw.measured[0] == 1            # local HBM gather was timed
    pick, pred = A.select_strategy(st, bw)
    tb = [[st.t_build_s[si][r] for r in range(C)] for si in range(4)]
    rpred, rpick = S.predict(ref, list(bw.alpha_s), list(bw.beta_Bps), tb)
    assert pick == rpick and np.allclose(pred, rpred, rtol=1e-9)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("strategy,C,fanouts", [("GDP", 1, (5, 5)), ("GDP", 2, (5, 5)), ("NFP", 2, (5, 5)),
                                                ("SNP", 4, (5, 5)), ("DNP", 4, (5, 5)), ("SNP", 2, (5, 5, 5)),
                                                ("NFP", 4, (12, 16))])
def test_layer_fwd_bwd_api(A, tiny, strategy, C, fanouts, dtype):
    """The standalone layer API of SURVEY §8(b) (sampler and upper layers are the
    user's black boxes): the caller samples each rank's batch with apt_sample, runs
    apt_layer_fwd(strategy, batch, store, W, bias) and feeds its own dL/dh1 to apt_layer_bwd
    -- h1 of every rank, dW1 and db1 (all-reduced; NFP assembled from the column-owned
    slices) against the oracle."""
    from oracle import strategy as S
    cfg, g, train = tiny
    cfg = cfg.replace(fanouts=fanouts)
    ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
    part = aptgen.partition(g.n, C)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    dt = A.DTYPE[dtype]
    fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    step = min(3, oracle.steps_per_epoch(len(train), C, cfg.batch) - 1)   # the last global batch is short
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    gb = oracle.global_batch(perm, step, C, cfg.batch)
    seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
    batches = [ctx.sample(gr, dev_i64(sd), len(sd), cfg.fanouts, cfg.sample_seed, step) for sd in seeds]
    batch = ctx.batch_group(batches) if C > 1 else batches[0]
    W, b = aptgen.weights(cfg)[0]
    d1 = W.shape[0]
    K = len(cfg.fanouts)
    rows = [len(oracle.sample_blocks(g, sd, cfg.fanouts, cfg.sample_seed, step)[K - 1].dst) for sd in seeds]
    h1 = torch.zeros((sum(rows), d1), dtype=torch.float32, device="cuda")
    saved = ctx.layer_fwd(A.STRATEGY[strategy], batch, fs, torch.as_tensor(W).cuda(), torch.as_tensor(b).cuda(), d1,
                          dt, h1)
    torch.cuda.synchronize()
    H = h1.cpu().numpy()
    Wr = oracle.bf16_round(W.astype(np.float64)) if dtype == "bf16" else W.astype(np.float64)
    rng = np.random.default_rng(C)
    dh = rng.normal(size=(sum(rows), d1)).astype(np.float32)
    dW = db = 0.0
    bW = bb = 0.0
    off = 0
    for r in range(C):
        blk = oracle.sample_blocks(g, seeds[r], cfg.fanouts, cfg.sample_seed, step)[K - 1]
        x = oracle.features(cfg.feat_seed, blk.src, cfg.dim)
        Zs = model.snp_partials(blk, x, part, C) if strategy == "SNP" else [oracle.aggregate(blk.indptr, blk.indices, x)]
        if dtype == "bf16":
            Zs = [oracle.bf16_round(z) for z in Zs]     # the bf16 rounding point of Z (SNP: of each partial, R5)
        pre = sum(z @ Wr.T for z in Zs) + b
        h = np.maximum(pre, 0.0)
        if dtype == "bf16":
            h = oracle.bf16_round(h)                      # the stored activation (R11)
        got = H[off:off + rows[r]]
        # T1 for the pre-activation (same operands on both sides), plus one bf16 flip of h
        Zabs = sum(np.abs(z) for z in Zs)
        sig = np.sqrt(Zs[0].shape[1]) * 2.0 ** -24 * (Zabs @ np.abs(Wr).T + np.abs(b))
        bound = 6 * sig + (2.0 ** -8 * np.abs(h) if dtype == "bf16" else 0.0)
        assert_close(got, h, dtype, f"h1 rank {r}", bound)
        # T3: the ReLU bit the GPU took where the pre-activation is within the band of zero
        on = got > 0
        amb = np.abs(pre) <= 6 * sig + (2.0 ** -8 * np.abs(pre) if dtype == "bf16" else 0.0)
        assert not ((on != (pre > 0)) & ~amb).any(), f"rank {r}: mask differs outside the ambiguity band"
        gpre = dh[off:off + rows[r]].astype(np.float64) * on
        if dtype == "bf16":
            gpre = oracle.bf16_round(gpre)                # reading R4: g rounded for tcgen05
        dW = dW + sum(gpre.T @ z for z in Zs)
        db = db + gpre.sum(0)
        bW = bW + t1(np.abs(gpre).T, Zabs, rows[r])
        bb = bb + t1(np.abs(gpre).T, np.ones(rows[r]), rows[r])
        off += rows[r]
    dW_dev = torch.zeros((d1, cfg.dim), dtype=torch.float32, device="cuda")
    db_dev = torch.zeros(d1, dtype=torch.float32, device="cuda")
    ctx.layer_bwd(saved, torch.as_tensor(dh).cuda(), dW_dev, db_dev)
    torch.cuda.synchronize()
    assert_close(dW_dev.cpu().numpy(), dW, "f32", "dW1", bW)     # emulated operands: fp32 bar + T1
    assert_close(db_dev.cpu().numpy(), db, "f32", "db1", bb)
    saved.close()


@pytest.mark.slow
def test_products_full_size_layer1_rows_vs_oracle(A, ctx):
    """BASELINE configs[1] at full size, in the bench's launch configuration (bf16, CUDA graph,
    pipelined GDP step): layer-1 Z of 300 sampled destinations recomputed one by one by the
    oracle (Floyd positions -> neighbour rows -> fp64 mean -> bf16) -- bit-exact under O4 -- and their
    h1 = ReLU(bf16(Z) bf16(W)^T + b) within the bf16 bar."""
    cfg = aptgen.CONFIGS["products"]
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    gr = ctx.graph_load(g.indptr, g.indices)
    fs = ctx.fstore_create(gr, A.GDP, A.BF16, cfg.dim, None, cfg.feat_seed)
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.BF16, 0.05, cfg.sample_seed, cfg.feat_seed, A.GDP,
                   labels)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    tr.set_epoch(train, 0)
    tr.use_graph(True)
    for step in range(3):
        tr.step(step, update=False)
    step = 2
    dst = tr.read("dst", 1)[:, 0].astype(np.int64)
    Z = tr.read("Z", 1)
    H = tr.read("H", 1)
    rng = np.random.default_rng(0)
    rows = rng.choice(len(dst), size=300, replace=False)
    K = len(cfg.fanouts)
    W1 = oracle.bf16_round(params[0][0].astype(np.float64))
    b1 = params[0][1].astype(np.float64)
    for i in rows:
        v = int(dst[i])
        deg = int(g.indptr[v + 1] - g.indptr[v])
        pos = oracle.sample_positions(v, deg, cfg.fanouts[0], cfg.sample_seed, step, K - 1)
        nbrs = g.indices[g.indptr[v] + pos].astype(np.int64)
        x = oracle.features(cfg.feat_seed, nbrs, cfg.dim)
        z = x.mean(axis=0) if len(nbrs) else np.zeros(cfg.dim)
        zb = oracle.bf16_round(z)                   # bf16 mode stores Z at its bf16 rounding point (O5)
        assert np.array_equal(Z[i], zb.astype(np.float32)), v
        h = np.maximum(zb @ W1.T + b1, 0)
        # same bf16 operands: fp32 accumulation (T1) and one bf16 rounding of h (2^-9, flip-wide)
        assert_close(H[i], h, "bf16", f"h1 of {v}", t1(np.abs(zb), np.abs(W1).T, cfg.dim) + 2.0 ** -8 * np.abs(h))


# ------------------------------------------------------------------ unified feature store tiers (NEXT #2)
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("frac,n_hot", [(0.5, 0), (0.3, 400), (1.0, 400)])
def test_tiered_store_rows_and_step(A, tiny, dtype, frac, n_hot):
    """HBM budget + pinned host tier + replicated hot rows: every row reads back bit-exact
    through each rank's view, and GDP / DNP / SNP steps at C = 2 still match the oracle."""
    cfg, g, train = tiny
    rng = np.random.default_rng(3)
    hot = rng.choice(g.n, size=n_hot, replace=False) if n_hot else None
    for strategy, C in (("GDP", 1), ("GDP", 2), ("DNP", 2), ("SNP", 2)):
        ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
        part = aptgen.partition(g.n, C)
        gr = ctx.graph_load(g.indptr, g.indices, part)
        fs = ctx.fstore_create(gr, A.GDP, A.DTYPE[dtype], cfg.dim, None, cfg.feat_seed, hbm_frac=frac, hot_ids=hot)
        if strategy == "GDP":
            ids = np.arange(g.n, dtype=np.int32)
            pitch = ((cfg.dim + 7) // 8 * 8) if dtype == "bf16" else ((cfg.dim + 3) // 4 * 4)
            esz = 2 if dtype == "bf16" else 4
            out = torch.zeros(g.n * pitch * esz, dtype=torch.uint8, device="cuda")
            torch.cuda.synchronize()
            ctx.gather(fs, torch.as_tensor(ids.astype(np.int64)).cuda(), g.n, out)
            torch.cuda.synchronize()
            raw = out.cpu().numpy()
            got = ((raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32) if dtype == "bf16"
                   else raw.view(np.float32)).reshape(g.n, pitch)[:, :cfg.dim]
            assert np.array_equal(got.astype(np.float64), oracle.features(cfg.feat_seed, ids.astype(np.int64), cfg.dim))
        dims = [cfg.dim] + [d for _, d in cfg.dims()]
        labels = aptgen.labels(cfg, g.n)
        tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.DTYPE[dtype], 0.1, cfg.sample_seed, cfg.feat_seed,
                       A.STRATEGY[strategy], labels)
        params = aptgen.weights(cfg)
        tr.set_params(params)
        tr.set_epoch(train, 0)
        tr.step(0, update=False)
        seeds, refs, bds = _strategy_ref(cfg, g, train, labels, params, strategy, C, 0, dtype, bounds=tr)
        for r in range(C):
            assert_close(tr.read("H", 1, rank=r), refs[r]["cache"]["h"][0], dtype, f"{strategy} C{C} H1 rank {r}",
                         bds[r]["H"][0])
        sb = sum_bounds(bds)
        for l in range(1, len(cfg.fanouts) + 1):
            assert_close(tr.read("dW", l, rank=0), sum(x["grads"][l - 1][0] for x in refs), dtype,
                         f"{strategy} C{C} dW{l}", sb["dW"][l - 1])


# ------------------------------------------------------------------ P:163 per-strategy caches (NEXT #2)
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("strategy,C,frac", [("GDP", 2, 0.1), ("SNP", 2, 0.3), ("DNP", 2, 0.2), ("DNP", 4, 0.05),
                                             ("GDP", 1, 0.02)])
def test_p163_cache_store(A, tiny, strategy, C, frac, dtype):
    """APT_CACHE_P163: every GPU's HBM holds its P:163 cache set (from the oracle's access
    counts), every row also on the pinned host; rows read back bit-exact through the view,
    the dry-run's per-tier counts equal the oracle's emulation under the same feature map
    (own cache / peer cache over NVLink / host), and the strategy's step still
    matches the oracle (the store only moves features)."""
    from oracle import strategy as S
    cfg, g, train = tiny
    part = aptgen.partition(g.n, C)
    counts = S.access_counts(g, train, cfg.fanouts, cfg.sample_seed, 0, C, cfg.batch, 2)
    budget = int(frac * g.n)
    ctx = A.Ctx(-1, C, 0) if C > 1 else A.Ctx(0, 1, 0)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    fs = ctx.fstore_create(gr, A.STRATEGY[strategy], A.DTYPE[dtype], cfg.dim, None, cfg.feat_seed, counts=counts,
                           cache_budget_rows=budget)
    ids = np.arange(g.n, dtype=np.int64)
    pitch = ((cfg.dim + 7) // 8 * 8) if dtype == "bf16" else ((cfg.dim + 3) // 4 * 4)
    esz = 2 if dtype == "bf16" else 4
    out = torch.zeros(g.n * pitch * esz, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    ctx.gather(fs, torch.as_tensor(ids).cuda(), g.n, out)
    torch.cuda.synchronize()
    raw = out.cpu().numpy()
    got = ((raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32) if dtype == "bf16"
           else raw.view(np.float32)).reshape(g.n, pitch)[:, :cfg.dim]
    assert np.array_equal(got.astype(np.float64), oracle.features(cfg.feat_seed, ids, cfg.dim))
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    labels = aptgen.labels(cfg, g.n)
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, A.DTYPE[dtype], 0.1, cfg.sample_seed, cfg.feat_seed,
                   A.STRATEGY[strategy], labels)
    params = aptgen.weights(cfg)
    tr.set_params(params)
    tr.set_epoch(train, 0)
    # dry-run tiers vs the oracle's feature map of the same caches
    st = tr.dryrun(2)
    sets = S.cache_sets(strategy, counts, part, C, budget, g.indptr, g.indices)
    tier = S.cached_store(sets, g.n)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    si = S.STRATEGIES.index(strategy)
    tot = [dict(rows_local=0, rows_peer=0, rows_host=0) for _ in range(C)]
    for step in range(st.steps):
        gb = oracle.global_batch(perm, step, C, cfg.batch)
        seeds = S.assign_seeds(strategy, gb, part, C, cfg.batch)
        blocks = [oracle.sample_blocks(g, sd, cfg.fanouts, cfg.sample_seed, step)[-1] for sd in seeds]
        for r, e in enumerate(S.emulate_layer1(strategy, blocks, part, C, cfg.dim, cfg.hidden, 4, 4, tier=tier)):
            for k in tot[r]:
                tot[r][k] += e[k]
    for r in range(C):
        for k in tot[r]:
            assert getattr(st, k)[si][r] == tot[r][k], (k, r, getattr(st, k)[si][r], tot[r][k])
    tr.step(0, update=False)
    seeds, refs, bds = _strategy_ref(cfg, g, train, labels, params, strategy, C, 0, dtype, bounds=tr)
    for r in range(C):
        assert_close(tr.read("H", 1, rank=r), refs[r]["cache"]["h"][0], dtype, f"H1 rank {r}", bds[r]["H"][0])
    sb = sum_bounds(bds)
    assert_close(tr.read("dW", 1, rank=0), sum(x["grads"][0][0] for x in refs), dtype, "dW1", sb["dW"][0])
