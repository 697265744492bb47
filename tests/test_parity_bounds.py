"""Self-check of the parity bounds (tests/parity_util.py, readings T1-T4) on the CPU.

The oracle's own bf16-mode evaluation (oracle/model.py rounding Z, W and hidden H to
bf16) is one valid bf16 evaluation of the definition, so it must lie within the "bf16u"
bounds of the unrounded fp64 evaluation; and the bounds must not be vacuous (median
well below the tensor's own rms), else the GPU parity tests would prove nothing.
"""
import numpy as np
import pytest

import aptgen
import oracle
from oracle import model
from parity_util import assert_close, reconcile, rms


@pytest.mark.parametrize("fanouts", [(5, 5), (5, 5, 5)])
def test_oracle_bf16_within_unrounded_bounds(tiny_cfg, tiny_graph, fanouts):
    cfg = tiny_cfg.replace(fanouts=fanouts)
    g = tiny_graph
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    seeds = oracle.epoch_perm(train, cfg.sample_seed, 0)[:cfg.batch]
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, 0)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in aptgen.weights(cfg)]
    ref_u = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), "f32")
    got = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), "bf16")
    K = len(blocks)
    ref_u, bd = reconcile(blocks, p64, ref_u, "bf16u", len(seeds), [got["cache"]["h"][l] for l in range(K - 1)])
    for l in range(K):
        assert_close(got["cache"]["h"][l], ref_u["cache"]["h"][l], "bf16u", f"H{l + 1}", bd["H"][l])
        assert_close(got["grads"][l][0], ref_u["grads"][l][0], "bf16u", f"dW{l + 1}", bd["dW"][l])
        assert_close(got["grads"][l][1], ref_u["grads"][l][1], "bf16u", f"db{l + 1}", bd["db"][l])
        # not vacuous: the typical allowance is a small fraction of the tensor's magnitude
        assert np.median(bd["dW"][l]) < 0.2 * rms(ref_u["grads"][l][0])
        assert np.median(bd["H"][l]) < 0.2 * rms(ref_u["cache"]["h"][l])


def test_bounds_catch_a_dropped_term(tiny_cfg, tiny_graph):
    """A plausible kernel bug -- the bias left out of layer 1 -- must fail the fp32 bar."""
    cfg, g = tiny_cfg, tiny_graph
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    seeds = oracle.epoch_perm(train, cfg.sample_seed, 0)[:cfg.batch]
    blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, 0)
    p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in aptgen.weights(cfg)]
    ref = model.train_step(blocks, cfg.feat_seed, cfg.dim, p64, labels[seeds], len(seeds), "f32")
    bad = [(p64[0][0], 0 * p64[0][1])] + p64[1:]
    got = model.train_step(blocks, cfg.feat_seed, cfg.dim, bad, labels[seeds], len(seeds), "f32")
    K = len(blocks)
    ref, bd = reconcile(blocks, p64, ref, "f32", len(seeds), [ref["cache"]["h"][l] for l in range(K - 1)])
    for dtype in ("f32", "bf16"):
        with pytest.raises(AssertionError):
            assert_close(got["cache"]["h"][0], ref["cache"]["h"][0], dtype, "H1", bd["H"][0])
        with pytest.raises(AssertionError):
            assert_close(got["grads"][1][0], ref["grads"][1][0], dtype, "dW2", bd["dW"][1])
