"""Partitioners (reading R10), -m "not gpu": the oracle pinned by
closed cases, and the library's host apt_partition bit-exact against it (no GPU)."""
import numpy as np
import pytest
import scipy.sparse as sp

import aptgen
from oracle import partition as P


def _cliques(k, s):
    edges = [(c * s + i, c * s + j) for c in range(k) for i in range(s) for j in range(i + 1, s)]
    return aptgen.graph_from_edges(k * s, edges)


def test_ldg_recovers_disjoint_cliques():
    g = _cliques(4, 25)
    part = P.ldg(g.indptr, g.indices, 4)
    assert P.cut_edges(g.indptr, g.indices, part) == 0
    assert sorted(np.bincount(part).tolist()) == [25] * 4
    assert np.array_equal(part, np.repeat(np.arange(4), 25))     # clique c -> part c (ties to the emptiest)


def test_cut_edges_brute_force_and_balance(tiny_graph):
    g = tiny_graph
    for C in (2, 4, 8):
        part = P.ldg(g.indptr, g.indices, C)
        cap = -(-105 * g.n // (100 * C))
        assert part.min() >= 0 and np.bincount(part, minlength=C).max() <= cap
        A = sp.csr_matrix((np.ones(g.nnz), g.indices, g.indptr), shape=(g.n, g.n))
        coo = A.tocoo()
        assert P.cut_edges(g.indptr, g.indices, part) == int((part[coo.row] != part[coo.col]).sum())


def test_random_partition_cut_and_ldg_beats_it(tiny_graph):
    # Fig. 11: a random partition cuts ~ (1 - 1/C) of the edges; the streaming
    # partitioner exploits locality and cuts fewer
    g = tiny_graph
    for C in (2, 4):
        rnd = P.random_part(g.n, C, seed=7)
        frac = P.cut_edges(g.indptr, g.indices, rnd) / g.nnz
        assert abs(frac - (1 - 1 / C)) < 0.03
        assert np.bincount(rnd, minlength=C).min() > 0.9 * g.n / C
        assert P.cut_edges(g.indptr, g.indices, P.ldg(g.indptr, g.indices, C)) < 0.8 * frac * g.nnz


def test_range_partition_is_the_generator_partition(tiny_graph):
    assert np.array_equal(P.range_part(tiny_graph.n, 4), aptgen.partition(tiny_graph.n, 4))


@pytest.mark.parametrize("C", [2, 4, 8])
def test_library_partitioner_bit_exact(tiny_graph, C):
    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
    g = tiny_graph
    for method, ref in (("range", P.range_part(g.n, C)), ("random", P.random_part(g.n, C, 7)),
                        ("ldg", P.ldg(g.indptr, g.indices, C))):
        part, cut = A.partition(g.indptr, g.indices, C, method, seed=7)
        assert np.array_equal(part, ref), method
        assert cut == P.cut_edges(g.indptr, g.indices, ref)
