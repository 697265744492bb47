// partition.cu -- graph partitioners for SNP / DNP.
//
// SNP and DNP partition the graph with an edge cut ("uses an edge-cut (e.g.,
// METIS [24])"), and the cut decides their virtual nodes (N_vs, N_vd,
// P:148) -- Fig. 11 shows what a poor partition costs.  METIS is
// an external library and too slow at these sizes (SURVEY §8(f) OUT), so APT's
// Prepare stage here offers:
//   APT_PART_RANGE   part(u) = floor(u * C / n): the generator's planted partition
//                    (aptgen plants communities in id ranges);
//   APT_PART_RANDOM  part(u) = Philox(seed; u) mod C: the random partition of the
//                    Fig. 11 ablation (cut ~ 1 - 1/C);
//   APT_PART_LDG     Linear Deterministic Greedy streaming (Stanton & Kliot, KDD'12),
//                    reading R10: nodes in ascending id; u goes to the partition p
//                    with size_p < cap maximising |N(u) ∩ P_p| * (cap - size_p)
//                    (integers: exact and reproducible), ties to the smaller
//                    size_p, then the smaller p; cap = ceil(1.05 n / C).
// Host code (the topology is on the host when the job is prepared); O(nnz + n C).
#include <cstdint>
#include <cstring>
#include <vector>

#include "common.cuh"
#include "runtime.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
}

extern "C" apt_status apt_partition(int64_t n, int64_t nnz, const int64_t* indptr, const int32_t* indices, int C,
                                    int method, uint64_t seed, int32_t* part, int64_t* cut_edges) {
  using apt::set_err;
  if (n < 1 || nnz < 0 || !indptr || (nnz > 0 && !indices) || !part || C < 1 || C > APT_MAX_RANKS ||
      method < APT_PART_RANGE || method > APT_PART_LDG || n >= (int64_t(1) << 31))
    return set_err(nullptr, APT_E_INVALID, "apt_partition: bad arguments");
  if (indptr[0] != 0 || indptr[n] != nnz) return set_err(nullptr, APT_E_INVALID, "apt_partition: indptr[0] / indptr[n]");
  if (method == APT_PART_RANGE) {
    for (int64_t u = 0; u < n; ++u) part[u] = int32_t((u * C) / n);
  } else if (method == APT_PART_RANDOM) {
    const uint2 key = apt::philox_key(seed, 0x50415254u /* "PART" */);
    for (int64_t u = 0; u < n; ++u) {
      const uint4 w = apt::philox(make_uint4(uint32_t(u), uint32_t(uint64_t(u) >> 32), 0u, 0u), key);
      part[u] = int32_t(w.x % uint32_t(C));
    }
  } else {
    const int64_t cap = (105 * n + 100 * int64_t(C) - 1) / (100 * int64_t(C));
    std::vector<int64_t> size(C, 0);
    for (int64_t u = 0; u < n; ++u) part[u] = -1;
    int64_t cnt[APT_MAX_RANKS];
    for (int64_t u = 0; u < n; ++u) {
      for (int p = 0; p < C; ++p) cnt[p] = 0;
      for (int64_t e = indptr[u]; e < indptr[u + 1]; ++e) {
        const int32_t v = indices[e];
        if (v < 0 || v >= n) return set_err(nullptr, APT_E_INVALID, "apt_partition: neighbour id out of range");
        if (part[v] >= 0) ++cnt[part[v]];
      }
      int best = -1;
      int64_t best_score = -1;
      for (int p = 0; p < C; ++p) {
        if (size[p] >= cap) continue;
        const int64_t sc = cnt[p] * (cap - size[p]);
        if (best < 0 || sc > best_score || (sc == best_score && size[p] < size[best])) {
          best = p;
          best_score = sc;
        }
      }
      part[u] = best;
      ++size[best];
    }
  }
  if (cut_edges) {   // directed CSR entries whose endpoints lie in different partitions
    int64_t cut = 0;
    for (int64_t u = 0; u < n; ++u)
      for (int64_t e = indptr[u]; e < indptr[u + 1]; ++e) cut += part[indices[e]] != part[u];
    *cut_edges = cut;
  }
  return APT_OK;
}
