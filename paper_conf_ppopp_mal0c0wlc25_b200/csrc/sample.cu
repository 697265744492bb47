// sample.cu -- S1-S3 of the hot path: seed selection, Philox-keyed fanout
// sampling (Fig. 2) and block compaction into CSR.
//
// B200 design:
//  * sampling: one warp per frontier node; lanes draw Philox words in parallel,
//    Floyd's sequential membership step is a ballot per draw, the ascending
//    order is a rank-by-count over shuffles (no sort), and the k chosen
//    neighbour ids are read with independent 4-byte loads.
//  * compaction: no sort and no hash table.  Node ids are < 2^31, so the set
//    "new neighbours not in dst" is a bitmap over all nodes (n/8 bytes: 300 KB
//    for 2.4M nodes, L2-resident); one popcount prefix scan over the bitmap
//    yields the ascending unique list and the global->local map in one pass.
//  * every count lives in device memory and every grid is sized by an upper
//    bound, so a whole step has no host sync and can be captured in a CUDA graph.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>

namespace apt {

// ------------------------------------------------------------- sampling ----
// S2 / reading O2: for frontier node v at hop h with fanout k:
//  deg <= k  -> all positions, no draws;
//  else Floyd: for t in 0..k-1, j = deg-k+t, w = word(t&3) of
//  Philox_SAMPLE(seed; {v_lo, v_hi, step, (h<<24)|(t>>2)}), r = (w*(j+1))>>32,
//  insert (r already chosen ? j : r); positions ascending.
template <int KS>  // KS = ceil(k/32) slots per lane
__global__ void __launch_bounds__(256) sample_kernel(const int64_t* __restrict__ indptr,
                                                     const int32_t* __restrict__ indices,
                                                     const int32_t* __restrict__ frontier,
                                                     const int32_t* __restrict__ n_frontier, int k,
                                                     uint2 key, const uint64_t* __restrict__ step_ptr,
                                                     int hop, int32_t* __restrict__ cnt,
                                                     int32_t* __restrict__ nbr) {
  const int lane = lane_id();
  const int64_t F = *n_frontier;
  const uint32_t step = uint32_t(*step_ptr);
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < F; i += nwarps) {
    const int v = frontier[i];
    const int64_t base = indptr[v];
    const int64_t deg = indptr[v + 1] - base;
    int32_t* out = nbr + i * k;
    if (deg <= k) {
      for (int q = lane; q < deg; q += 32) out[q] = indices[base + q];
      if (lane == 0) cnt[i] = int32_t(deg);
      continue;
    }
    uint32_t chosen[KS];
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      const int t_me = s * 32 + lane;
      uint32_t r_me = 0;
      if (t_me < k) {
        const uint4 w = philox(make_uint4(uint32_t(v), 0u, step, (uint32_t(hop) << 24) | uint32_t(t_me >> 2)), key);
        const uint64_t j = uint64_t(deg - k + t_me);
        r_me = uint32_t((uint64_t(word_of(w, t_me & 3)) * (j + 1)) >> 32);
      }
      chosen[s] = 0xFFFFFFFFu;
      const int n_t = min(32, k - s * 32);
      for (int tt = 0; tt < n_t; ++tt) {
        const uint32_t r = __shfl_sync(0xffffffffu, r_me, tt);
        bool hit = false;
#pragma unroll
        for (int s2 = 0; s2 < KS; ++s2)
          if (s2 < s || (s2 == s && lane < tt)) hit |= (chosen[s2] == r);
        const bool member = __any_sync(0xffffffffu, hit);
        if (lane == tt) chosen[s] = member ? uint32_t(deg - k + s * 32 + tt) : r;
      }
    }
    // ascending order: rank of every chosen position among all k (all distinct)
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      const int t_me = s * 32 + lane;
      int rank = 0;
#pragma unroll
      for (int s2 = 0; s2 < KS; ++s2) {
        const int n_t = min(32, k - s2 * 32);
        for (int tt = 0; tt < n_t; ++tt) {
          const uint32_t o = __shfl_sync(0xffffffffu, chosen[s2], tt);
          rank += (o < chosen[s]) ? 1 : 0;
        }
      }
      if (t_me < k) out[rank] = indices[base + chosen[s]];
    }
    if (lane == 0) cnt[i] = k;
  }
}

cudaError_t launch_sample(const SampleArgs& a, cudaStream_t st) {
  const int threads = 256;
  const int64_t warps = a.max_frontier;
  int64_t blocks = ceil_div(warps * 32, threads);
  blocks = std::max<int64_t>(1, std::min<int64_t>(blocks, 148 * 16));
  const int ks = int(ceil_div(a.k, 32));
#define APT_SAMPLE_CASE(KS)                                                                      \
  case KS:                                                                                       \
    sample_kernel<KS><<<blocks, threads, 0, st>>>(a.indptr, a.indices, a.frontier, a.n_frontier, \
                                                  a.k, a.key, a.step, a.hop, a.cnt, a.nbr);      \
    break;
  switch (ks) {
    APT_SAMPLE_CASE(1)
    APT_SAMPLE_CASE(2)
    APT_SAMPLE_CASE(4)
    APT_SAMPLE_CASE(8)
    case 3:
      sample_kernel<4><<<blocks, threads, 0, st>>>(a.indptr, a.indices, a.frontier, a.n_frontier,
                                                   a.k, a.key, a.step, a.hop, a.cnt, a.nbr);
      break;
    default:
      sample_kernel<8><<<blocks, threads, 0, st>>>(a.indptr, a.indices, a.frontier, a.n_frontier,
                                                   a.k, a.key, a.step, a.hop, a.cnt, a.nbr);
  }
#undef APT_SAMPLE_CASE
  return cudaGetLastError();
}

// ------------------------------------------------------ device-wide scan ----
// Three-kernel reduce-then-scan over int32 values: partials -> spine -> emit.
constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;

template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* total) {
  __shared__ T warp_tot[kScanThreads / 32];
  const int lane = lane_id(), wid = threadIdx.x >> 5;
  T incl = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T n = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += n;
  }
  if (lane == 31) warp_tot[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    T w = lane < kScanThreads / 32 ? warp_tot[lane] : T(0);
    T wi = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      T n = __shfl_up_sync(0xffffffffu, wi, o);
      if (lane >= o) wi += n;
    }
    if (lane < kScanThreads / 32) warp_tot[lane] = wi - w;
    if (lane == kScanThreads / 32 - 1) *total = wi;
  }
  __syncthreads();
  T r = warp_tot[wid] + incl - v;
  __syncthreads();
  return r;
}

template <class Op>
__global__ void __launch_bounds__(kScanThreads) scan_partials(Op op, int32_t* partials) {
  const int64_t n = op.size();
  const int64_t base = int64_t(blockIdx.x) * kScanTile + int64_t(threadIdx.x) * kScanItems;
  int32_t s = 0;
#pragma unroll
  for (int j = 0; j < kScanItems; ++j)
    if (base + j < n) s += op.value(base + j);
  __shared__ int32_t tot;
  block_exclusive_scan<int32_t>(s, &tot);
  if (threadIdx.x == 0) partials[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(1024) scan_spine(int32_t* partials, int nb) {
  __shared__ int32_t carry_s;
  __shared__ int32_t wsum[32];
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (int off = 0; off < nb; off += 1024) {
    const int i = off + threadIdx.x;
    const int32_t v = i < nb ? partials[i] : 0;
    const int lane = lane_id(), wid = threadIdx.x >> 5;
    int32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int32_t n = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += n;
    }
    if (lane == 31) wsum[wid] = incl;
    __syncthreads();
    if (wid == 0) {
      int32_t w = wsum[lane], wi = w;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int32_t n = __shfl_up_sync(0xffffffffu, wi, o);
        if (lane >= o) wi += n;
      }
      wsum[lane] = wi - w;
    }
    __syncthreads();
    const int32_t carry = carry_s;
    const int32_t excl = carry + wsum[wid] + incl - v;
    if (i < nb) partials[i] = excl;
    __syncthreads();
    if (threadIdx.x == 1023) carry_s = excl + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) partials[nb] = carry_s;   // grand total
}

template <class Op>
__global__ void __launch_bounds__(kScanThreads) scan_emit(Op op, const int32_t* partials, int nb) {
  const int64_t n = op.size();
  const int64_t base = int64_t(blockIdx.x) * kScanTile + int64_t(threadIdx.x) * kScanItems;
  int32_t vals[kScanItems];
  int32_t s = 0;
#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    vals[j] = (base + j < n) ? op.value(base + j) : 0;
    s += vals[j];
  }
  __shared__ int32_t tot;
  int32_t excl = block_exclusive_scan<int32_t>(s, &tot) + partials[blockIdx.x];
#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    if (base + j < n) op.emit(base + j, excl, vals[j]);
    excl += vals[j];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) op.finish(partials[nb]);
}

template <class Op>
static cudaError_t run_scan(const Op& op, int64_t max_n, int32_t* partials, cudaStream_t st) {
  const int nb = int(std::max<int64_t>(1, ceil_div(max_n, kScanTile)));
  scan_partials<Op><<<nb, kScanThreads, 0, st>>>(op, partials);
  scan_spine<<<1, 1024, 0, st>>>(partials, nb);
  scan_emit<Op><<<nb, kScanThreads, 0, st>>>(op, partials, nb);
  return cudaGetLastError();
}

// --------------------------------------------------------- compaction ----
// S3 / reading O3: src = dst ++ ascending(unique(nbrs) \ dst); indptr = scan(cnt);
// indices[e] = position of nbr[e] in src.

__global__ void mark_dst_kernel(const int32_t* __restrict__ dst, const int32_t* __restrict__ n_dst,
                                uint32_t* __restrict__ dst_bm, int32_t* __restrict__ pos) {
  const int64_t F = *n_dst;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < F; i += int64_t(gridDim.x) * blockDim.x) {
    const int v = dst[i];
    atomicOr(dst_bm + (v >> 5), 1u << (v & 31));
    pos[v] = int32_t(i);
  }
}

__global__ void mark_new_kernel(const int32_t* __restrict__ cnt, const int32_t* __restrict__ nbr,
                                const int32_t* __restrict__ n_dst, int k,
                                const uint32_t* __restrict__ dst_bm, uint32_t* __restrict__ new_bm) {
  const int64_t slots = int64_t(*n_dst) * k;
  for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < slots; s += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = s / k;
    const int q = int(s - i * k);
    if (q >= cnt[i]) continue;
    const int u = nbr[s];
    const uint32_t bit = 1u << (u & 31);
    if (dst_bm[u >> 5] & bit) continue;
    if (!(__ldcg(new_bm + (u >> 5)) & bit)) atomicOr(new_bm + (u >> 5), bit);
  }
}

struct BitmapScanOp {
  uint32_t* new_bm;
  int64_t n_words;
  const int32_t* n_dst;
  int32_t* src;
  int32_t* pos;
  int32_t* n_src;
  __device__ int64_t size() const { return n_words; }
  __device__ int32_t value(int64_t w) const { return __popc(new_bm[w]); }
  __device__ void emit(int64_t w, int32_t excl, int32_t val) const {
    if (!val) return;
    uint32_t word = new_bm[w];
    int32_t idx = *n_dst + excl;
    while (word) {
      const int b = __ffs(word) - 1;
      word &= word - 1;
      const int u = int(w * 32 + b);
      src[idx] = u;
      pos[u] = idx;
      ++idx;
    }
    new_bm[w] = 0u;   // leave the bitmap clean for the next hop
  }
  __device__ void finish(int32_t total) const { *n_src = *n_dst + total; }
};

struct CntScanOp {
  const int32_t* cnt;
  const int32_t* n_dst;
  int32_t* indptr;
  int32_t* n_edges;
  __device__ int64_t size() const { return *n_dst; }
  __device__ int32_t value(int64_t i) const { return cnt[i]; }
  __device__ void emit(int64_t i, int32_t excl, int32_t) const { indptr[i] = excl; }
  __device__ void finish(int32_t total) const {
    indptr[*n_dst] = total;
    *n_edges = total;
  }
};

__global__ void map_indices_kernel(const int32_t* __restrict__ dst, const int32_t* __restrict__ cnt,
                                   const int32_t* __restrict__ nbr, const int32_t* __restrict__ n_dst,
                                   int k, const int32_t* __restrict__ indptr,
                                   const int32_t* __restrict__ pos, int32_t* __restrict__ indices,
                                   uint32_t* __restrict__ dst_bm) {
  const int64_t slots = int64_t(*n_dst) * k;
  for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < slots; s += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = s / k;
    const int q = int(s - i * k);
    if (q == 0) {
      const int v = dst[i];
      atomicAnd(dst_bm + (v >> 5), ~(1u << (v & 31)));
    }
    if (q >= cnt[i]) continue;
    indices[indptr[i] + q] = pos[nbr[s]];
  }
}

static int64_t grid_for(int64_t n, int threads) {
  return std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, threads), 148 * 32));
}

cudaError_t launch_compact(const CompactArgs& a, cudaStream_t st) {
  const int T = 256;
  mark_dst_kernel<<<grid_for(a.max_dst, T), T, 0, st>>>(a.dst, a.n_dst, a.dst_bm, a.pos);
  mark_new_kernel<<<grid_for(a.max_dst * a.k, T), T, 0, st>>>(a.cnt, a.nbr, a.n_dst, a.k, a.dst_bm, a.new_bm);
  // src ids are written after the dst prefix by the bitmap scan; the prefix
  // itself is a copy of dst (the frontier).
  cudaError_t e = cudaMemcpyAsync(a.src, a.dst, sizeof(int32_t) * size_t(a.max_dst), cudaMemcpyDeviceToDevice, st);
  if (e != cudaSuccess) return e;
  BitmapScanOp bop{a.new_bm, a.n_words, a.n_dst, a.src, a.pos, a.n_src};
  e = run_scan(bop, a.n_words, a.partials, st);
  if (e != cudaSuccess) return e;
  CntScanOp cop{a.cnt, a.n_dst, a.indptr, a.n_edges};
  e = run_scan(cop, a.max_dst, a.partials2, st);
  if (e != cudaSuccess) return e;
  map_indices_kernel<<<grid_for(a.max_dst * a.k, T), T, 0, st>>>(a.dst, a.cnt, a.nbr, a.n_dst, a.k, a.indptr,
                                                                  a.pos, a.indices, a.dst_bm);
  return cudaGetLastError();
}

// ------------------------------------------------------------ S1 seeds ----
// GDP/NFP: contiguous chunk r of global batch t (perm[t*C*B + r*B ...]);
// SNP/DNP: the global batch's seeds with part(s) == r, in permutation order
// (O1, P:163 last sentence).  One CTA (global batch <= C*B <= 8*2048).
__global__ void __launch_bounds__(1024) select_seeds_kernel(const int32_t* __restrict__ perm, int64_t n_train,
                                                            const uint64_t* __restrict__ step_ptr, int64_t steps_per_epoch,
                                                            int world, int rank, int batch, int by_part,
                                                            const int32_t* __restrict__ part,
                                                            int32_t* __restrict__ seeds, int32_t* __restrict__ n_seeds,
                                                            int32_t* __restrict__ n_global) {
  const int64_t t = int64_t(*step_ptr % uint64_t(steps_per_epoch));
  const int64_t g0 = t * int64_t(world) * batch;
  int64_t gn = n_train - g0;
  if (gn > int64_t(world) * batch) gn = int64_t(world) * batch;
  if (gn < 0) gn = 0;
  if (!by_part) {
    const int64_t s0 = gn < int64_t(rank) * batch ? gn : int64_t(rank) * batch;
    const int64_t s1 = gn < int64_t(rank + 1) * batch ? gn : int64_t(rank + 1) * batch;
    for (int64_t i = threadIdx.x; i < s1 - s0; i += blockDim.x) seeds[i] = perm[g0 + s0 + i];
    if (threadIdx.x == 0) { *n_seeds = int32_t(s1 - s0); *n_global = int32_t(gn); }
    return;
  }
  __shared__ int32_t carry;
  __shared__ int32_t wtot[32];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t off = 0; off < gn; off += blockDim.x) {
    const int64_t i = off + threadIdx.x;
    const int32_t s = i < gn ? perm[g0 + i] : 0;
    const int keep = (i < gn && part[s] == rank) ? 1 : 0;
    const unsigned bal = __ballot_sync(0xffffffffu, keep);
    const int lane = lane_id(), wid = threadIdx.x >> 5;
    if (lane == 0) wtot[wid] = __popc(bal);
    __syncthreads();
    if (threadIdx.x == 0) {
      int acc = 0;
      for (int w = 0; w < int(blockDim.x >> 5); ++w) { int c = wtot[w]; wtot[w] = acc; acc += c; }
    }
    __syncthreads();
    const int32_t c0 = carry;
    if (keep) seeds[c0 + wtot[wid] + __popc(bal & ((1u << lane) - 1u))] = s;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = c0 + wtot[wid] + __popc(bal);
    __syncthreads();
  }
  if (threadIdx.x == 0) { *n_seeds = carry; *n_global = int32_t(gn); }
}

cudaError_t launch_select_seeds(const SeedArgs& a, cudaStream_t st) {
  select_seeds_kernel<<<1, 1024, 0, st>>>(a.perm, a.n_train, a.step, a.steps_per_epoch, a.world, a.rank,
                                          a.batch, a.by_part, a.part, a.seeds, a.n_seeds, a.n_global);
  return cudaGetLastError();
}

// Epoch permutation keys (O1): key(u) = Philox_PERM(seed;{u_lo,u_hi,epoch,0}).(w0 | w1<<32)
__global__ void perm_keys_kernel(const int32_t* __restrict__ train, int64_t n, uint2 key, uint32_t epoch,
                                 uint64_t* __restrict__ keys) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const uint4 w = philox(make_uint4(uint32_t(train[i]), 0u, epoch, 0u), key);
    keys[i] = uint64_t(w.x) | (uint64_t(w.y) << 32);
  }
}

cudaError_t launch_perm_keys(const int32_t* train, int64_t n, uint64_t seed, uint64_t epoch, uint64_t* keys,
                             cudaStream_t st) {
  perm_keys_kernel<<<grid_for(n, 256), 256, 0, st>>>(train, n, philox_key(seed, kDomPerm), uint32_t(epoch), keys);
  return cudaGetLastError();
}

}  // namespace apt
