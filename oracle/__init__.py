"""oracle -- plain, slow CPU ORACLE for APT's sampled-subgraph step.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA path; the only common module is
``aptgen`` (seeded input generators, none of the method's arithmetic).

Layout:
  apt_oracle.c   Philox4x32-10 (O0), epoch permutation (O1), Floyd sampler
                 (O2), block compaction (O3), features (O4), mean aggregation
                 and its backward (O5) -- single-threaded C, fp64.
  __init__.py    ctypes wrapper + the K-hop sampling driver.
  model.py       fp64 GraphSAGE forward/backward, CE loss (Eq. 1).
  strategy.py    per-rank emulation of GDP/NFP/SNP/DNP, their
                 counted volumes and the Eq. 2 cost model.

Parity status per function is listed in DESIGN.md §Oracle.  The sampler's
bit pattern is "parity unpinned" by the paper (it fixes no RNG): it is
pinned only by our reading O2 plus the Random123 KATs.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

DOMAIN = {"SAMPLE": 0x53414D50, "FEAT": 0x46454154, "PERM": 0x5045524D}


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "apt_oracle.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", src, "-o", _LIB])
    return _LIB


def _p(a):
    return a.ctypes.data


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        vp, i64, u64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int
        L.orc_philox4x32_10.argtypes = [vp, vp, vp]
        L.orc_perm_key.argtypes = [u64, u64, i64]
        L.orc_perm_key.restype = u64
        L.orc_epoch_perm.argtypes = [vp, i64, u64, u64, vp]
        L.orc_sample_positions.argtypes = [i64, i64, i32, u64, u64, i32, vp, vp]
        L.orc_sample_hop.argtypes = [vp, vp, vp, i64, i32, u64, u64, i32, vp, vp]
        L.orc_compact.argtypes = [vp, i64, vp, vp, i32, vp, vp, vp]
        L.orc_compact.restype = i64
        L.orc_feature.argtypes = [u64, i64, i32]
        L.orc_feature.restype = ctypes.c_double
        L.orc_features.argtypes = [u64, vp, i64, i32, vp]
        L.orc_aggregate.argtypes = [vp, vp, i64, vp, i32, vp]
        L.orc_aggregate_bwd.argtypes = [vp, vp, i64, vp, i32, vp]
        _lib = L
    return _lib


# ------------------------------------------------------------------ O0 ----
def philox(ctr, key):
    c = np.ascontiguousarray(ctr, np.uint32)
    k = np.ascontiguousarray(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(_p(c), _p(k), _p(out))
    return out


# ------------------------------------------------------------------ O1 ----
def epoch_perm(train: np.ndarray, seed: int, epoch: int) -> np.ndarray:
    train = np.ascontiguousarray(train, np.int64)
    out = np.empty_like(train)
    lib().orc_epoch_perm(_p(train), len(train), seed, epoch, _p(out))
    return out


def steps_per_epoch(n_train: int, world: int, batch: int) -> int:
    return -(-n_train // (world * batch))


def global_batch(perm: np.ndarray, t: int, world: int, batch: int) -> np.ndarray:
    """Global batch t = perm[t*C*B, (t+1)*C*B) (last one short)  (O1)."""
    return perm[t * world * batch:(t + 1) * world * batch]


# ------------------------------------------------------------------ O2 ----
def sample_positions(v: int, deg: int, k: int, seed: int, step: int, hop: int) -> np.ndarray:
    pos = np.zeros(max(k, 1), np.int64)
    cnt = ctypes.c_int(0)
    lib().orc_sample_positions(v, deg, k, seed, step, hop, _p(pos), ctypes.addressof(cnt))
    return pos[:cnt.value].copy()


def sample_hop(graph, frontier: np.ndarray, k: int, seed: int, step: int, hop: int):
    frontier = np.ascontiguousarray(frontier, np.int64)
    F = len(frontier)
    cnt = np.zeros(F, np.int32)
    nbr = np.full(max(F * k, 1), -1, np.int64)
    lib().orc_sample_hop(_p(graph.indptr), _p(graph.indices), _p(frontier), F, k, seed, step, hop,
                         _p(cnt), _p(nbr))
    return cnt, nbr[:F * k]


# ------------------------------------------------------------------ O3 ----
def compact(dst: np.ndarray, cnt: np.ndarray, nbr: np.ndarray, k: int):
    dst = np.ascontiguousarray(dst, np.int64)
    F = len(dst)
    src = np.empty(max(F * (1 + k), 1), np.int64)
    indptr = np.zeros(F + 1, np.int64)
    E = int(cnt.sum())
    indices = np.zeros(max(E, 1), np.int32)
    cnt = np.ascontiguousarray(cnt, np.int32)
    nbr = np.ascontiguousarray(nbr, np.int64)
    n_src = lib().orc_compact(_p(dst), F, _p(cnt), _p(nbr), k, _p(src), _p(indptr), _p(indices))
    return src[:n_src].copy(), indptr, indices[:E].copy()


class Block:
    """A sampled bipartite block: dst prefix of src, CSR over local ids."""

    def __init__(self, hop, dst, src, indptr, indices, cnt, nbr, k):
        self.hop, self.dst, self.src = hop, dst, src
        self.indptr, self.indices = indptr, indices
        self.cnt, self.nbr, self.k = cnt, nbr, k

    @property
    def n_dst(self):
        return len(self.dst)

    @property
    def n_src(self):
        return len(self.src)

    @property
    def n_edges(self):
        return int(self.indptr[-1])

    def deg(self):
        return np.diff(self.indptr)


def sample_blocks(graph, seeds: np.ndarray, fanouts, seed: int, step: int):
    """K-hop node-wise sampling: blocks[h] for hop h = 0..K-1 (h=0 at the
    seeds).  Hop h uses fanouts[K-1-h]; layer l's block is blocks[K-l]  (O2/O3, Z6)."""
    K = len(fanouts)
    blocks = []
    frontier = np.ascontiguousarray(seeds, np.int64)
    for h in range(K):
        k = int(fanouts[K - 1 - h])
        cnt, nbr = sample_hop(graph, frontier, k, seed, step, h)
        src, indptr, indices = compact(frontier, cnt, nbr, k)
        blocks.append(Block(h, frontier, src, indptr, indices, cnt, nbr, k))
        frontier = src
    return blocks


# ------------------------------------------------------------------ O4 ----
def features(seed: int, ids: np.ndarray, d: int) -> np.ndarray:
    ids = np.ascontiguousarray(ids, np.int64)
    out = np.empty((len(ids), d), np.float64)
    lib().orc_features(seed, _p(ids), len(ids), d, _p(out))
    return out


# ------------------------------------------------------------------ O5 ----
def aggregate(indptr, indices, x_src: np.ndarray) -> np.ndarray:
    n_dst = len(indptr) - 1
    x_src = np.ascontiguousarray(x_src, np.float64)
    d = x_src.shape[1]
    z = np.zeros((n_dst, d), np.float64)
    lib().orc_aggregate(_p(np.ascontiguousarray(indptr, np.int64)),
                        _p(np.ascontiguousarray(indices, np.int32)), n_dst, _p(x_src), d, _p(z))
    return z


def aggregate_bwd(indptr, indices, dz: np.ndarray, n_src: int) -> np.ndarray:
    n_dst = len(indptr) - 1
    dz = np.ascontiguousarray(dz, np.float64)
    d = dz.shape[1]
    dx = np.zeros((n_src, d), np.float64)
    lib().orc_aggregate_bwd(_p(np.ascontiguousarray(indptr, np.int64)),
                            _p(np.ascontiguousarray(indices, np.int32)), n_dst, _p(dz), d, _p(dx))
    return dx


def bf16_round(x) -> np.ndarray:
    """fp64 -> fp32 (RN) -> bf16 (RNE), returned as float64 (the bf16-mode rounding points, O5)."""
    f = np.ascontiguousarray(x, np.float32)
    b = f.view(np.uint32).astype(np.uint64)
    b = (b + 0x7FFF + ((b >> 16) & 1)) & 0xFFFF0000
    return b.astype(np.uint32).view(np.float32).astype(np.float64)
