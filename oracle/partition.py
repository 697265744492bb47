"""Edge-cut partitioners -- ORACLE (test infrastructure only).

SNP and DNP need an edge-cut partition ("uses an edge-cut (e.g., METIS [24])",
P:128); its quality sets their virtual-node counts (Fig. 11
compares METIS with a random partition).  Plain Python, written from the
definitions (reading R10 for LDG):
  range   part(u) = floor(u C / n)
  random  part(u) = Philox_PART(seed; {u_lo, u_hi, 0, 0}).word0 mod C
  ldg     linear deterministic greedy streaming (Stanton & Kliot, KDD'12): nodes in
          ascending id; u goes to the p with size_p < cap maximising
          |N(u) ∩ P_p| * (cap - size_p); ties -> smaller size_p, then smaller p;
          cap = ceil(1.05 n / C).
"""
from __future__ import annotations

import numpy as np

from . import philox

PART_DOMAIN = 0x50415254   # "PART"


def range_part(n: int, C: int) -> np.ndarray:
    return np.array([(u * C) // n for u in range(n)], np.int32)


def random_part(n: int, C: int, seed: int) -> np.ndarray:
    key = [seed & 0xFFFFFFFF, ((seed >> 32) & 0xFFFFFFFF) ^ PART_DOMAIN]
    return np.array([int(philox([u & 0xFFFFFFFF, u >> 32, 0, 0], key)[0]) % C for u in range(n)], np.int32)


def ldg(indptr, indices, C: int) -> np.ndarray:
    n = len(indptr) - 1
    cap = -(-105 * n // (100 * C))
    part = np.full(n, -1, np.int64)
    size = [0] * C
    for u in range(n):
        cnt = [0] * C
        for v in indices[indptr[u]:indptr[u + 1]]:
            if part[v] >= 0:
                cnt[part[v]] += 1
        best, best_score = -1, -1
        for p in range(C):
            if size[p] >= cap:
                continue
            sc = cnt[p] * (cap - size[p])
            if best < 0 or sc > best_score or (sc == best_score and size[p] < size[best]):
                best, best_score = p, sc
        part[u] = best
        size[best] += 1
    return part.astype(np.int32)


def cut_edges(indptr, indices, part) -> int:
    """CSR entries (u, v) with part[u] != part[v] (each undirected cut edge twice)."""
    rows = np.repeat(np.arange(len(indptr) - 1), np.diff(indptr))
    return int((np.asarray(part)[rows] != np.asarray(part)[np.asarray(indices)]).sum())
