/*
 * aptgen/rmat.c -- seeded synthetic INPUT generator (graph topology only).
 *
 * This file holds none of APT's arithmetic: it only manufactures the input
 * graph that both the CUDA path and the CPU oracle consume (the one module
 * the two are allowed to share).
 *
 * Recipe:
 *   * R-MAT (Chakrabarti et al. 2004): every undirected edge e draws `scale`
 *     quadrant choices.  The top `planted` levels use a planted-partition
 *     quadrant distribution (P(same bit) = p_same, symmetric), so a range
 *     partition into 2^planted parts has a cut fraction of 1 - p_same^planted
 *     and equal part masses.  The remaining levels use (a, b, c, d).
 *   * ids are scaled to [0, n): id' = floor(id * n / 2^scale)  (monotone, so
 *     the range partition survives).
 *   * the graph is symmetrised, self loops and duplicates are dropped, and
 *     rows are sorted ascending (CSR: int64 indptr, int32 indices).
 *   The random stream is a counter-based splitmix64 hash of (seed, e, level);
 *   it is independent of the Philox generator the method itself uses.
 *
 * Build: gcc -O3 -fopenmp -shared -fPIC aptgen/rmat.c -o aptgen/libaptgen.so
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static inline double u01(uint64_t seed, uint64_t a, uint64_t b) {
  uint64_t h = mix64(seed ^ mix64(a * 0x100000001B3ull + mix64(b + 0x51ED27ull)));
  return (double)(h >> 11) * (1.0 / 9007199254740992.0);
}

typedef struct {
  int64_t n, nnz;
  int64_t *indptr;
  int32_t *indices;
} aptgen_csr;

static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

/* Generate an R-MAT graph and return a heap CSR (free with aptgen_free). */
aptgen_csr *aptgen_rmat(int64_t n, int64_t m, int scale, double a, double b,
                        double c, int planted, double p_same, uint64_t seed,
                        int threads) {
  if (n <= 0 || m < 0 || scale < 1 || scale > 40) return NULL;
  if (threads > 0) omp_set_num_threads(threads);
  int32_t *eu = (int32_t *)malloc(sizeof(int32_t) * (size_t)(m ? m : 1));
  int32_t *ev = (int32_t *)malloc(sizeof(int32_t) * (size_t)(m ? m : 1));
  int64_t *deg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  if (!eu || !ev || !deg) return NULL;
  const double ps2 = p_same * 0.5, pd2 = (1.0 - p_same) * 0.5;

#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < m; ++e) {
    uint64_t u = 0, v = 0;
    for (int l = 0; l < scale; ++l) {
      double r = u01(seed, (uint64_t)e, (uint64_t)l);
      int bu, bv;
      if (l < planted) {
        if (r < ps2) { bu = 0; bv = 0; }
        else if (r < 2 * ps2) { bu = 1; bv = 1; }
        else if (r < 2 * ps2 + pd2) { bu = 0; bv = 1; }
        else { bu = 1; bv = 0; }
      } else {
        if (r < a) { bu = 0; bv = 0; }
        else if (r < a + b) { bu = 0; bv = 1; }
        else if (r < a + b + c) { bu = 1; bv = 0; }
        else { bu = 1; bv = 1; }
      }
      u = (u << 1) | (uint64_t)bu;
      v = (v << 1) | (uint64_t)bv;
    }
    /* monotone scaling to [0, n) */
    u = (uint64_t)(((unsigned __int128)u * (uint64_t)n) >> scale);
    v = (uint64_t)(((unsigned __int128)v * (uint64_t)n) >> scale);
    eu[e] = (int32_t)u;
    ev[e] = (int32_t)v;
    if (u != v) {
      __atomic_fetch_add(&deg[u], 1, __ATOMIC_RELAXED);
      __atomic_fetch_add(&deg[v], 1, __ATOMIC_RELAXED);
    }
  }

  /* exclusive scan of degrees -> provisional row starts */
  int64_t *start = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
  start[0] = 0;
  for (int64_t i = 0; i < n; ++i) start[i + 1] = start[i] + deg[i];
  int64_t total = start[n];
  int32_t *tmp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(total ? total : 1));
  int64_t *cur = deg; /* reuse as cursor */
  memcpy(cur, start, sizeof(int64_t) * (size_t)n);

#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < m; ++e) {
    int32_t u = eu[e], v = ev[e];
    if (u == v) continue;
    int64_t pu = __atomic_fetch_add(&cur[u], 1, __ATOMIC_RELAXED);
    int64_t pv = __atomic_fetch_add(&cur[v], 1, __ATOMIC_RELAXED);
    tmp[pu] = v;
    tmp[pv] = u;
  }
  free(eu);
  free(ev);

  /* sort + dedupe every row (deterministic regardless of scatter order) */
  int64_t *ndeg = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    int64_t s = start[i], len = start[i + 1] - s;
    if (len > 1) qsort(tmp + s, (size_t)len, sizeof(int32_t), cmp_i32);
    int64_t w = 0;
    for (int64_t j = 0; j < len; ++j)
      if (j == 0 || tmp[s + j] != tmp[s + j - 1]) tmp[s + w++] = tmp[s + j];
    ndeg[i] = w;
  }
  aptgen_csr *g = (aptgen_csr *)malloc(sizeof(aptgen_csr));
  g->n = n;
  g->indptr = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
  g->indptr[0] = 0;
  for (int64_t i = 0; i < n; ++i) g->indptr[i + 1] = g->indptr[i] + ndeg[i];
  g->nnz = g->indptr[n];
  g->indices = (int32_t *)malloc(sizeof(int32_t) * (size_t)(g->nnz ? g->nnz : 1));
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    memcpy(g->indices + g->indptr[i], tmp + start[i], sizeof(int32_t) * (size_t)ndeg[i]);
  free(tmp);
  free(start);
  free(ndeg);
  free(deg);
  return g;
}

int64_t aptgen_n(const aptgen_csr *g) { return g->n; }
int64_t aptgen_nnz(const aptgen_csr *g) { return g->nnz; }
void aptgen_copy(const aptgen_csr *g, int64_t *indptr, int32_t *indices) {
  memcpy(indptr, g->indptr, sizeof(int64_t) * ((size_t)g->n + 1));
  memcpy(indices, g->indices, sizeof(int32_t) * (size_t)g->nnz);
}
void aptgen_free(aptgen_csr *g) {
  if (!g) return;
  free(g->indptr);
  free(g->indices);
  free(g);
}

/* Seeded per-node hash in [0,1): used for train-set membership and labels. */
void aptgen_node_u01(uint64_t seed, int64_t n, double *out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = u01(seed, (uint64_t)i, 0x7A11ull);
}
