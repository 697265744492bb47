"""aptgen -- seeded synthetic INPUT generators shared by the CUDA path and the oracle.

This module is the only code both sides may use.  It
holds none of APT's arithmetic: it makes the graph topology (R-MAT with a
planted range partition), the train set, the labels, the partition vector
and the initial weights.  Node features and the sampler's random draws are
NOT made here: both sides implement the same counter-based Philox generator
for those.

Config shapes follow BASELINE.json ``configs`` and SURVEY.md §8(d):
  tiny      10k nodes / 100k undirected edges, d=64, SAGE 64->32->16, fanout [5,5], B=256
  products  2.4M / 62M, d=100, SAGE 100->256->256->47, fanout [10,10,10], B=1024
  papers    111M / 1.6B, d in {64,256}, SAGE d->32->32->172
  friendster 65M / 1.8B, d=256, SAGE 256->h->h->64, h in {8,32,128}
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libaptgen.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the generator (plain gcc, OpenMP)."""
    src = os.path.join(_HERE, "rmat.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", src, "-o", _LIB])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.aptgen_rmat.restype = ctypes.c_void_p
        lib.aptgen_rmat.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_double,
                                    ctypes.c_double, ctypes.c_double, ctypes.c_int, ctypes.c_double,
                                    ctypes.c_uint64, ctypes.c_int]
        lib.aptgen_n.restype = ctypes.c_int64
        lib.aptgen_n.argtypes = [ctypes.c_void_p]
        lib.aptgen_nnz.restype = ctypes.c_int64
        lib.aptgen_nnz.argtypes = [ctypes.c_void_p]
        lib.aptgen_copy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.aptgen_free.argtypes = [ctypes.c_void_p]
        lib.aptgen_node_u01.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p]
        _lib = lib
    return _lib


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    n: int                 # nodes
    m: int                 # undirected R-MAT edges drawn (before dedupe)
    scale: int             # R-MAT levels, 2^scale >= n
    abc: tuple             # R-MAT (a, b, c); d = 1 - a - b - c
    dim: int               # input feature dim d
    hidden: int            # hidden dim d'
    n_classes: int
    fanouts: tuple         # fanouts[l-1] is layer l's fanout (DGL convention)
    batch: int             # seeds per GPU (B)
    train_frac: float
    planted: int = 3       # planted-partition levels (log2 C_max)
    p_same: float = 0.93   # P(same top bit) per planted level
    graph_seed: int = 1
    feat_seed: int = 2
    sample_seed: int = 3
    weight_seed: int = 4
    label_seed: int = 5

    @property
    def n_layers(self) -> int:
        return len(self.fanouts)

    def dims(self):
        """[(d_in, d_out)] for every layer (layer 1 first)."""
        ds = [self.dim] + [self.hidden] * (self.n_layers - 1) + [self.n_classes]
        return [(ds[i], ds[i + 1]) for i in range(self.n_layers)]

    def replace(self, **kw) -> "Config":
        return dataclasses.replace(self, **kw)


GRAPH500 = (0.57, 0.19, 0.19)
FLAT = (0.45, 0.22, 0.22)

CONFIGS = {
    "tiny": Config("tiny", 10_000, 100_000, 14, GRAPH500, 64, 32, 16, (5, 5), 256, 0.10),
    "products": Config("products", 2_400_000, 62_000_000, 22, GRAPH500, 100, 256, 47,
                       (10, 10, 10), 1024, 0.08),
    "papers": Config("papers", 111_000_000, 1_600_000_000, 27, GRAPH500, 64, 32, 172,
                     (10, 10, 10), 1024, 0.0109),
    "friendster": Config("friendster", 65_000_000, 1_800_000_000, 26, FLAT, 256, 32, 64,
                         (10, 10, 10), 1024, 0.01),
}


@dataclasses.dataclass
class Graph:
    n: int
    indptr: np.ndarray   # int64 [n+1]
    indices: np.ndarray  # int32 [nnz], rows ascending, symmetric, no self loops / duplicates

    @property
    def nnz(self) -> int:
        return int(self.indptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.indptr)


def make_graph(cfg: Config, threads: int = 0) -> Graph:
    lib = _load()
    a, b, c = cfg.abc
    h = lib.aptgen_rmat(cfg.n, cfg.m, cfg.scale, a, b, c, cfg.planted, cfg.p_same,
                        cfg.graph_seed, threads)
    if not h:
        raise RuntimeError("aptgen_rmat failed")
    try:
        n, nnz = lib.aptgen_n(h), lib.aptgen_nnz(h)
        indptr = np.empty(n + 1, np.int64)
        indices = np.empty(nnz, np.int32)
        lib.aptgen_copy(h, indptr.ctypes.data, indices.ctypes.data)
    finally:
        lib.aptgen_free(h)
    return Graph(n, indptr, indices)


def graph_from_edges(n: int, edges) -> Graph:
    """Symmetric CSR from an explicit undirected edge list (hand-built fixtures)."""
    adj = [set() for _ in range(n)]
    for u, v in edges:
        if u != v:
            adj[u].add(v)
            adj[v].add(u)
    indptr = np.zeros(n + 1, np.int64)
    for i in range(n):
        indptr[i + 1] = indptr[i] + len(adj[i])
    indices = np.array([v for i in range(n) for v in sorted(adj[i])], np.int32)
    return Graph(n, indptr, indices)


def node_u01(seed: int, n: int) -> np.ndarray:
    out = np.empty(n, np.float64)
    _load().aptgen_node_u01(seed, n, out.ctypes.data)
    return out


def train_nodes(graph: Graph, cfg: Config) -> np.ndarray:
    """Ascending int64 train ids: non-isolated nodes with hash < train_frac (Z11, Z27)."""
    u = node_u01(cfg.graph_seed ^ 0x7121, graph.n)
    return np.nonzero((u < cfg.train_frac) & (graph.degrees() > 0))[0].astype(np.int64)


def labels(cfg: Config, n: int) -> np.ndarray:
    u = node_u01(cfg.label_seed, n)
    return np.minimum((u * cfg.n_classes).astype(np.int32), cfg.n_classes - 1)


def partition(n: int, world: int) -> np.ndarray:
    """Range partition part(u) = floor(u * C / n): the planted R-MAT partition (§8(d))."""
    return ((np.arange(n, dtype=np.int64) * world) // n).astype(np.int32)


def weights(cfg: Config):
    """Initial [(W [d_out x d_in] fp32, b [d_out] fp32)] for every layer, layer 1 first."""
    rng = np.random.default_rng(cfg.weight_seed)
    out = []
    for d_in, d_out in cfg.dims():
        s = 1.0 / np.sqrt(d_in)
        W = rng.uniform(-s, s, size=(d_out, d_in)).astype(np.float32)
        b = rng.uniform(-0.1, 0.1, size=(d_out,)).astype(np.float32)
        out.append((W, b))
    return out
