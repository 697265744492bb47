/*
 * oracle/apt_oracle.c -- plain, slow, single-threaded CPU ORACLE for APT's
 * sampled-subgraph step (Ma et al., "Adaptive Parallel Training for Graph
 * Neural Networks", PPoPP'25).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code with the CUDA path (paper_conf_ppopp_mal0c0wlc25_b200/csrc)
 * and never includes any of its headers.
 *
 * Citations "P:<line>" are lines of /root/reference/PAPER.md; "O<k>" / "Z<k>"
 * are the readings in SURVEY.md §8(c), restated in DESIGN.md §Readings.
 *
 * Pins (tests/test_oracle_pins.py): Random123 known-answer vectors for
 * Philox; exact subset enumeration / chi-square / pairwise inclusion for the
 * sampler; brute-force set arithmetic for compaction; the dense D^-1 A X
 * special case for aggregation.  "Sampler bits" are parity-unpinned by the
 * paper (it fixes no RNG): pinned only by our spec O2 + the KATs.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- O0 ---- */
/* Philox4x32-10 (Salmon et al., SC'11).  The paper fixes no RNG (P:108 is
 * silent, reading Z2); this counter-based generator lets every GPU and this
 * oracle draw the same neighbours for the same (node, hop, step).          */
#define PHILOX_M0 0xD2511F53u
#define PHILOX_M1 0xCD9E8D57u
#define PHILOX_W0 0x9E3779B9u
#define PHILOX_W1 0xBB67AE85u

void orc_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
  uint32_t k0 = key_in[0], k1 = key_in[1];
  for (int round = 0; round < 10; ++round) {
    if (round > 0) { k0 += PHILOX_W0; k1 += PHILOX_W1; }
    uint64_t p0 = (uint64_t)PHILOX_M0 * (uint64_t)c0;
    uint64_t p1 = (uint64_t)PHILOX_M1 * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* Domain separation: key = (seed_lo, seed_hi ^ DOMAIN). */
#define DOM_SAMPLE 0x53414D50u
#define DOM_FEAT   0x46454154u
#define DOM_PERM   0x5045524Du

static void make_key(uint64_t seed, uint32_t domain, uint32_t key[2]) {
  key[0] = (uint32_t)seed;
  key[1] = (uint32_t)(seed >> 32) ^ domain;
}

/* ---------------------------------------------------------------- O1 ---- */
/* Epoch permutation ("an epoch covers all seeds"):
 * key(u) = Philox_PERM(seed; {u_lo, u_hi, epoch, 0}).word0 | word1 << 32,
 * perm = train sorted ascending by (key, u).                              */
uint64_t orc_perm_key(uint64_t seed, uint64_t epoch, int64_t u) {
  uint32_t key[2], ctr[4], out[4];
  make_key(seed, DOM_PERM, key);
  ctr[0] = (uint32_t)(uint64_t)u;
  ctr[1] = (uint32_t)((uint64_t)u >> 32);
  ctr[2] = (uint32_t)epoch;
  ctr[3] = 0;
  orc_philox4x32_10(ctr, key, out);
  return (uint64_t)out[0] | ((uint64_t)out[1] << 32);
}

typedef struct { uint64_t key; int64_t u; } perm_item;
static int cmp_perm(const void *a, const void *b) {
  const perm_item *x = (const perm_item *)a, *y = (const perm_item *)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  return (x->u > y->u) - (x->u < y->u);
}

void orc_epoch_perm(const int64_t *train, int64_t n_train, uint64_t seed, uint64_t epoch,
                    int64_t *perm) {
  perm_item *it = (perm_item *)malloc(sizeof(perm_item) * (size_t)(n_train ? n_train : 1));
  for (int64_t i = 0; i < n_train; ++i) {
    it[i].u = train[i];
    it[i].key = orc_perm_key(seed, epoch, train[i]);
  }
  qsort(it, (size_t)n_train, sizeof(perm_item), cmp_perm);
  for (int64_t i = 0; i < n_train; ++i) perm[i] = it[i].u;
  free(it);
}

/* ---------------------------------------------------------------- O2 ---- */
/* Node-wise uniform fanout sampling without replacement (Fig. 2;
 * Z1 without replacement, Z3 multiply-shift, Z4 Floyd + ascending positions).
 * For frontier node v at hop h with fanout k:
 *   deg <= k : positions 0..deg-1, no draws;
 *   else Floyd: S = {}; for t in 0..k-1: j = deg-k+t;
 *        w = word (t&3) of Philox_SAMPLE(seed; {v_lo, v_hi, step, (h<<24)|(t>>2)})
 *        r = floor(w * (j+1) / 2^32); insert (r in S ? j : r).
 * Output: cnt[i], and nbr[i*k + 0..cnt-1] = indices[indptr[v] + pos] with the
 * chosen positions sorted ascending.                                       */
static int cmp_i64(const void *a, const void *b) {
  int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
  return (x > y) - (x < y);
}

void orc_sample_positions(int64_t v, int64_t deg, int k, uint64_t seed, uint64_t step, int hop,
                          int64_t *pos /* k */, int *cnt_out) {
  if (deg <= k) {
    for (int64_t p = 0; p < deg; ++p) pos[p] = p;
    *cnt_out = (int)deg;
    return;
  }
  uint32_t key[2], ctr[4], out[4];
  make_key(seed, DOM_SAMPLE, key);
  int n = 0;
  for (int t = 0; t < k; ++t) {
    ctr[0] = (uint32_t)(uint64_t)v;
    ctr[1] = (uint32_t)((uint64_t)v >> 32);
    ctr[2] = (uint32_t)step;
    ctr[3] = ((uint32_t)hop << 24) | ((uint32_t)t >> 2);
    orc_philox4x32_10(ctr, key, out);
    uint32_t w = out[t & 3];
    int64_t j = deg - k + t;
    int64_t r = (int64_t)(((uint64_t)w * (uint64_t)(j + 1)) >> 32);
    int member = 0;
    for (int q = 0; q < n; ++q)
      if (pos[q] == r) { member = 1; break; }
    pos[n++] = member ? j : r;
  }
  qsort(pos, (size_t)n, sizeof(int64_t), cmp_i64);
  *cnt_out = n;
}

void orc_sample_hop(const int64_t *indptr, const int32_t *indices, const int64_t *frontier,
                    int64_t F, int k, uint64_t seed, uint64_t step, int hop, int32_t *cnt,
                    int64_t *nbr /* F*k */) {
  int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)k);
  for (int64_t i = 0; i < F; ++i) {
    int64_t v = frontier[i];
    int64_t deg = indptr[v + 1] - indptr[v];
    int c = 0;
    orc_sample_positions(v, deg, k, seed, step, hop, pos, &c);
    cnt[i] = c;
    for (int q = 0; q < c; ++q) nbr[i * k + q] = indices[indptr[v] + pos[q]];
    for (int q = c; q < k; ++q) nbr[i * k + q] = -1;
  }
  free(pos);
}

/* ---------------------------------------------------------------- O3 ---- */
/* Block compaction ("bipartite graph that consists of source and destination
 * nodes"; Z7 node order): src = dst ++ sort_ascending(unique(nbrs) \ dst),
 * indptr = cumulative cnt in dst order, indices[e] = position of nbr in src.
 * Returns n_src.  src_out capacity >= F*(1+k).                              */
static int64_t find_sorted(const int64_t *a, int64_t n, int64_t x) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) / 2;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return (lo < n && a[lo] == x) ? lo : -1;
}

typedef struct { int64_t id; int64_t pos; } idpos;
static int cmp_idpos(const void *a, const void *b) {
  const idpos *x = (const idpos *)a, *y = (const idpos *)b;
  return (x->id > y->id) - (x->id < y->id);
}

int64_t orc_compact(const int64_t *dst, int64_t F, const int32_t *cnt, const int64_t *nbr, int k,
                    int64_t *src_out, int64_t *indptr_out, int32_t *indices_out) {
  /* dst lookup table (dst ids are unique) */
  idpos *dl = (idpos *)malloc(sizeof(idpos) * (size_t)(F ? F : 1));
  for (int64_t i = 0; i < F; ++i) { dl[i].id = dst[i]; dl[i].pos = i; }
  qsort(dl, (size_t)F, sizeof(idpos), cmp_idpos);
  int64_t *dsorted = (int64_t *)malloc(sizeof(int64_t) * (size_t)(F ? F : 1));
  for (int64_t i = 0; i < F; ++i) dsorted[i] = dl[i].id;

  /* candidate new ids = all sampled neighbours not in dst */
  int64_t E = 0;
  for (int64_t i = 0; i < F; ++i) E += cnt[i];
  int64_t *cand = (int64_t *)malloc(sizeof(int64_t) * (size_t)(E ? E : 1));
  int64_t nc = 0;
  for (int64_t i = 0; i < F; ++i)
    for (int q = 0; q < cnt[i]; ++q) {
      int64_t u = nbr[i * k + q];
      if (find_sorted(dsorted, F, u) < 0) cand[nc++] = u;
    }
  qsort(cand, (size_t)nc, sizeof(int64_t), cmp_i64);
  int64_t nu = 0;
  for (int64_t i = 0; i < nc; ++i)
    if (i == 0 || cand[i] != cand[i - 1]) cand[nu++] = cand[i];

  for (int64_t i = 0; i < F; ++i) src_out[i] = dst[i];
  for (int64_t i = 0; i < nu; ++i) src_out[F + i] = cand[i];

  indptr_out[0] = 0;
  int64_t e = 0;
  for (int64_t i = 0; i < F; ++i) {
    for (int q = 0; q < cnt[i]; ++q) {
      int64_t u = nbr[i * k + q];
      int64_t p = find_sorted(dsorted, F, u);
      if (p >= 0) p = dl[p].pos;
      else p = F + find_sorted(cand, nu, u);
      indices_out[e++] = (int32_t)p;
    }
    indptr_out[i + 1] = e;
  }
  free(dl);
  free(dsorted);
  free(cand);
  return F + nu;
}

/* ---------------------------------------------------------------- O4 ---- */
/* Synthetic input features (the paper's h_v^0; values are our input
 * recipe): x[u][j] = (int8)(Philox_FEAT(seed; {u_lo,u_hi,j>>2,0}).word(j&3)
 * & 0xFF) / 64.  Every value is k/64 with |k| <= 128: exact in bf16 & fp32. */
double orc_feature(uint64_t seed, int64_t u, int j) {
  uint32_t key[2], ctr[4], out[4];
  make_key(seed, DOM_FEAT, key);
  ctr[0] = (uint32_t)(uint64_t)u;
  ctr[1] = (uint32_t)((uint64_t)u >> 32);
  ctr[2] = (uint32_t)(j >> 2);
  ctr[3] = 0;
  orc_philox4x32_10(ctr, key, out);
  int8_t b = (int8_t)(out[j & 3] & 0xFFu);
  return (double)b / 64.0;
}

void orc_features(uint64_t seed, const int64_t *ids, int64_t n, int d, double *out) {
  for (int64_t i = 0; i < n; ++i)
    for (int j = 0; j < d; ++j) out[i * d + j] = orc_feature(seed, ids[i], j);
}

/* ---------------------------------------------------------------- O5 ---- */
/* GraphSAGE mean aggregation ("GraphSAGE uses the mean aggregation
 * function"; Eq. 1 P:100 AGG over sampled N(v)):
 *   z[v] = (1/deg_s(v)) * sum_{e in row v} x[indices[e]],  z = 0 if deg_s = 0 (Z11).
 * fp64 throughout.                                                          */
void orc_aggregate(const int64_t *indptr, const int32_t *indices, int64_t n_dst,
                   const double *x_src, int d, double *z) {
  for (int64_t v = 0; v < n_dst; ++v) {
    int64_t s = indptr[v], e = indptr[v + 1];
    for (int j = 0; j < d; ++j) {
      double acc = 0.0;
      for (int64_t q = s; q < e; ++q) acc += x_src[(int64_t)indices[q] * d + j];
      z[v * d + j] = (e > s) ? acc / (double)(e - s) : 0.0;
    }
  }
}

/* Backward of the mean (O5): dx[indices[e]] += dz[v] / deg_s(v).            */
void orc_aggregate_bwd(const int64_t *indptr, const int32_t *indices, int64_t n_dst,
                       const double *dz, int d, double *dx_src) {
  for (int64_t v = 0; v < n_dst; ++v) {
    int64_t s = indptr[v], e = indptr[v + 1];
    if (e == s) continue;
    double inv = 1.0 / (double)(e - s);
    for (int64_t q = s; q < e; ++q)
      for (int j = 0; j < d; ++j) dx_src[(int64_t)indices[q] * d + j] += dz[v * d + j] * inv;
  }
}
