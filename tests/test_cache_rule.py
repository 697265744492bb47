"""P:163's per-strategy cache configuration (-m "not gpu"): the library's host routine
apt_cache_sets equals the oracle's rule (oracle/strategy.py cache_sets, itself pinned by
brute force in test_oracle_strategy.py) for every strategy, bit for bit."""
import numpy as np
import pytest

import aptgen
from oracle import strategy as S


@pytest.mark.parametrize("strategy", ["GDP", "NFP", "SNP", "DNP"])
@pytest.mark.parametrize("budget", [0, 1, 333, 20000])
def test_cache_sets_library_equals_oracle(tiny_graph, tiny_cfg, strategy, budget):
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    g, C = tiny_graph, 4
    part = aptgen.partition(g.n, C)
    counts = S.access_counts(g, aptgen.train_nodes(g, tiny_cfg), tiny_cfg.fanouts, tiny_cfg.sample_seed, 0, C,
                             tiny_cfg.batch, 2)
    got = A.cache_sets(g.indptr, g.indices, part, C, A.STRATEGY[strategy], counts, budget)
    ref = S.cache_sets(strategy, counts, part, C, budget, g.indptr, g.indices)
    for r in range(C):
        assert np.array_equal(got[r], ref[r]), (strategy, r)
