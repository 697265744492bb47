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
__global__ void __launch_bounds__(256, (KS <= 2 ? 8 : 4)) sample_kernel(const int64_t* __restrict__ indptr,
                                                     const int32_t* __restrict__ indices,
                                                     const int32_t* __restrict__ frontier,
                                                     const int32_t* __restrict__ n_frontier, int k,
                                                     uint2 key, const uint64_t* __restrict__ step_ptr,
                                                     int hop, int32_t* __restrict__ cnt,
                                                     int32_t* __restrict__ nbr) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t F = *n_frontier;
  const uint32_t step = uint32_t(*step_ptr);
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  // software pipeline over the warp's frontier nodes: the next node's CSR bounds and
  // the id after it are loaded while the current node draws and gathers, so a node's
  // chain starts at its neighbour loads (frontier -> indptr -> indices was 3 deep)
  int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  int v_cur = i < F ? frontier[i] : 0;
  int64_t b0 = i < F ? indptr[v_cur] : 0, b1 = i < F ? indptr[v_cur + 1] : 0;
  int v_nxt = i + nwarps < F ? frontier[i + nwarps] : 0;
  for (; i < F; i += nwarps) {
    const int v = v_cur;
    const int64_t base = b0;
    const int64_t deg = b1 - b0;
    if (i + nwarps < F) { b0 = indptr[v_nxt]; b1 = indptr[v_nxt + 1]; }
    v_cur = v_nxt;
    v_nxt = i + 2 * nwarps < F ? frontier[i + 2 * nwarps] : 0;
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

// Fanout <= 16: two frontier nodes per warp, one per 16-lane half (k of 16 lanes busy
// instead of k of 32), the same draws and the same Floyd / ranking steps as
// sample_kernel with every shuffle confined to the half (bit-identical output).
__global__ void __launch_bounds__(256, 6) sample_g16_kernel(const int64_t* __restrict__ indptr,
                                                            const int32_t* __restrict__ indices,
                                                            const int32_t* __restrict__ frontier,
                                                            const int32_t* __restrict__ n_frontier, int k,
                                                            uint2 key, const uint64_t* __restrict__ step_ptr,
                                                            int hop, int32_t* __restrict__ cnt,
                                                            int32_t* __restrict__ nbr) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int g = lane >> 4, l = lane & 15;
  const uint32_t gmask = g ? 0xFFFF0000u : 0x0000FFFFu;
  const int64_t F = *n_frontier;
  const uint32_t step = uint32_t(*step_ptr);
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  const int64_t stride = 2 * nwarps;
  // node of this half: i = 2 * warp + g; the next node's CSR bounds and the id after
  // it are loaded one iteration ahead (as in sample_kernel)
  int64_t i = ((int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5) * 2 + g;
  int v_cur = i < F ? frontier[i] : 0;
  int64_t b0 = i < F ? indptr[v_cur] : 0, b1 = i < F ? indptr[v_cur + 1] : 0;
  int v_nxt = i + stride < F ? frontier[i + stride] : 0;
  for (int64_t i0 = i - g; i0 < F; i0 += stride, i += stride) {   // warp-uniform loop
    const bool valid = i < F;
    const int v = v_cur;
    const int64_t base = b0;
    const int64_t deg = valid ? b1 - b0 : 0;
    if (i + stride < F) { b0 = indptr[v_nxt]; b1 = indptr[v_nxt + 1]; }
    v_cur = v_nxt;
    v_nxt = i + 2 * stride < F ? frontier[i + 2 * stride] : 0;
    int32_t* out = nbr + i * k;
    const bool small = deg <= k;
    // draws (only the halves that sample use them)
    uint32_t r_me = 0;
    if (valid && !small && l < k) {
      const uint4 w = philox(make_uint4(uint32_t(v), 0u, step, (uint32_t(hop) << 24) | uint32_t(l >> 2)), key);
      const uint64_t j = uint64_t(deg - k + l);
      r_me = uint32_t((uint64_t(word_of(w, l & 3)) * (j + 1)) >> 32);
    }
    uint32_t chosen = 0xFFFFFFFFu;
    for (int tt = 0; tt < k; ++tt) {   // Floyd's membership step, one draw at a time
      const uint32_t r = __shfl_sync(0xffffffffu, r_me, tt, 16);
      const bool hit = l < tt && chosen == r;
      const bool member = (__ballot_sync(0xffffffffu, hit) & gmask) != 0u;
      if (l == tt) chosen = member ? uint32_t(deg - k + tt) : r;
    }
    int rank = 0;
    for (int tt = 0; tt < k; ++tt) {
      const uint32_t o = __shfl_sync(0xffffffffu, chosen, tt, 16);
      rank += (o < chosen) ? 1 : 0;
    }
    if (!valid) continue;
    if (small) {
      for (int q = l; q < deg; q += 16) out[q] = indices[base + q];
      if (l == 0) cnt[i] = int32_t(deg);
    } else {
      if (l < k) out[rank] = indices[base + chosen];
      if (l == 0) cnt[i] = k;
    }
  }
}

cudaError_t launch_sample(const SampleArgs& a, cudaStream_t st) {
  const int threads = 256;
  const int64_t warps = a.max_frontier;
  int64_t blocks = ceil_div(warps * 32, threads);
  blocks = std::max<int64_t>(1, std::min<int64_t>(blocks, a.grid_cap > 0 ? a.grid_cap : int64_t(num_sms()) * 16));
  const int ks = int(ceil_div(a.k, 32));
  static const int g16 = [] { const char* v = std::getenv("APT_SAMPLE_G16"); return v ? atoi(v) : 1; }();
  if (g16 && a.k <= 16) {
    int64_t b2 = ceil_div(ceil_div(a.max_frontier, 2) * 32, threads);
    b2 = std::max<int64_t>(1, std::min<int64_t>(b2, a.grid_cap > 0 ? a.grid_cap : int64_t(num_sms()) * 16));
    launch_pdl(sample_g16_kernel, dim3(b2), dim3(threads), 0, st, a.indptr, a.indices, a.frontier, a.n_frontier, a.k,
               a.key, a.step, a.hop, a.cnt, a.nbr);
    return cudaGetLastError();
  }
#define APT_SAMPLE_CASE(KS)                                                                      \
  case KS:                                                                                       \
    launch_pdl(sample_kernel<KS>, dim3(blocks), dim3(threads), 0, st, a.indptr, a.indices, a.frontier, a.n_frontier, \
                                                  a.k, a.key, a.step, a.hop, a.cnt, a.nbr);      \
    break;
  switch (ks) {
    APT_SAMPLE_CASE(1)
    APT_SAMPLE_CASE(2)
    APT_SAMPLE_CASE(4)
    APT_SAMPLE_CASE(8)
    case 3:
      launch_pdl(sample_kernel<4>, dim3(blocks), dim3(threads), 0, st, a.indptr, a.indices, a.frontier, a.n_frontier,
                                                   a.k, a.key, a.step, a.hop, a.cnt, a.nbr);
      break;
    default:
      launch_pdl(sample_kernel<8>, dim3(blocks), dim3(threads), 0, st, a.indptr, a.indices, a.frontier, a.n_frontier,
                                                   a.k, a.key, a.step, a.hop, a.cnt, a.nbr);
  }
#undef APT_SAMPLE_CASE
  return cudaGetLastError();
}

// ------------------------------------------------------ device-wide scan ----
// Three-kernel reduce-then-scan over int32 values: partials -> spine -> emit.
constexpr int kScanThreads = 256;
constexpr int kScanItems = 4;   // 1 024-word tiles: 8 -> 4 doubles the CTAs of the look-back scans
static_assert((kScanThreads * kScanItems) % kScanWsTile == 0, "scan workspace granularity");
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

// --------------------------------------------------------- compaction ----
// S3 / reading O3: src = dst ++ ascending(unique(nbrs) \ dst); indptr = scan(cnt);
// indices[e] = position of nbr[e] in src.

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
                                   uint32_t* __restrict__ dst_bm, int32_t* __restrict__ csc_cnt,
                                   uint64_t* __restrict__ csc_st, int csc_nb, int32_t* __restrict__ csc_ticket) {
  APT_PDL_PROLOGUE();
  if (csc_st) {
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i <= csc_nb; i += int64_t(gridDim.x) * blockDim.x) {
      if (i < csc_nb) csc_st[i] = 0;
      else *csc_ticket = 0;
    }
  }
  const int64_t slots = int64_t(*n_dst) * k;
  for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < slots; s += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = s / k;
    const int q = int(s - i * k);
    if (q == 0) {
      const int v = dst[i];
      atomicAnd(dst_bm + (v >> 5), ~(1u << (v & 31)));
    }
    if (q >= cnt[i]) continue;
    const int u = pos[nbr[s]];
    indices[indptr[i] + q] = u;
    if (csc_cnt) atomicAdd(csc_cnt + u, 1);   // in-degree of local source u (block transpose)
  }
}

static int64_t grid_for(int64_t n, int threads) {
  return grid_cap(ceil_div(n, threads), 32);
}

// Fused compaction, three launches per hop:
//  1. mark: dst bits + pos[dst] + the dst prefix of src, every sampled neighbour's bit
//     (no exclusion yet: a block cannot know the dst bitmap is complete), clears the
//     scan state of step 2;
//  2. one single-pass scan (decoupled look-back; tickets give blocks their order) over
//     two domains at once: the words of (new & ~dst) -> ascending new ids, their
//     positions and n_src; the counts -> indptr and n_edges;
//  3. map_indices (above): indices[e] = pos[nbr[e]], and the dst bits are cleared.
__global__ void compact_mark_kernel(const int32_t* __restrict__ dst, const int32_t* __restrict__ n_dst,
                                    const int32_t* __restrict__ cnt, const int32_t* __restrict__ nbr, int k,
                                    uint32_t* __restrict__ dst_bm, uint32_t* __restrict__ new_bm,
                                    int32_t* __restrict__ pos, int32_t* __restrict__ src, uint64_t* __restrict__ stA,
                                    int nbA, uint64_t* __restrict__ stB, int nbB, int32_t* __restrict__ ticket) {
  APT_PDL_PROLOGUE();
  const int64_t F = *n_dst;
  const int64_t tid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x, nth = int64_t(gridDim.x) * blockDim.x;
  for (int64_t i = tid; i < nbA + nbB + 1; i += nth) {
    if (i < nbA) stA[i] = 0;
    else if (i < nbA + nbB) stB[i - nbA] = 0;
    else *ticket = 0;
  }
  for (int64_t i = tid; i < F; i += nth) {
    const int v = dst[i];
    atomicOr(dst_bm + (v >> 5), 1u << (v & 31));
    pos[v] = int32_t(i);
    src[i] = v;
  }
  const int64_t slots = F * k;
  for (int64_t s = tid; s < slots; s += nth) {
    const int64_t i = s / k;
    const int q = int(s - i * k);
    if (q >= cnt[i]) continue;
    const int u = nbr[s];
    const uint32_t bit = 1u << (u & 31);
    if (!(__ldcg(new_bm + (u >> 5)) & bit)) atomicOr(new_bm + (u >> 5), bit);
  }
}

__device__ __forceinline__ void st_release_gpu(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Decoupled look-back for block `b` of a chain, by one warp: publish the block
// aggregate, then inspect the 32 nearest predecessors at once (each lane spins on
// one slot until it carries a flag), sum back to the nearest inclusive prefix, and
// move the window 32 blocks back if none was inclusive yet; finally publish the
// block's own inclusive prefix.  All lanes of warp 0 call it; all return the prefix.
__device__ int32_t chain_prefix(uint64_t* st, int b, int32_t agg) {
  constexpr uint64_t kAgg = 1ull << 32, kIncl = 2ull << 32, kFlags = 3ull << 32;
  const int lane = lane_id();
  if (b == 0) {
    if (lane == 0) st_release_gpu(st, kIncl | uint32_t(agg));
    return 0;
  }
  if (lane == 0) st_release_gpu(st + b, kAgg | uint32_t(agg));
  int32_t excl = 0;
  for (int end = b;; end -= 32) {
    const int j = end - 1 - lane;
    uint64_t w = 0;
    if (j >= 0) {
      do { w = ld_acquire_gpu(st + j); } while (!(w & kFlags));
    }
    const unsigned incl = __ballot_sync(0xffffffffu, j >= 0 && (w & kFlags) == kIncl);
    const int stop = incl ? __ffs(incl) - 1 : 31;
    excl += warp_sum((j >= 0 && lane <= stop) ? int32_t(uint32_t(w)) : 0);
    if (incl) break;
  }
  if (lane == 0) st_release_gpu(st + b, kIncl | uint32_t(excl + agg));
  return excl;
}

template <class Op>
__device__ void scan_tile(const Op& op, uint64_t* st, int b, int nb) {
  const int64_t n = op.size();
  // the grid is sized by the capacity (the count lives on the device): tiles past the
  // data take no part in the look-back chain, and the last tile WITH data (tile 0 of an
  // empty scan) publishes the total -- at the products shape the hop-1 count scan has
  // 7 real tiles out of 121
  const int nb_real = n > 0 ? int(std::min<int64_t>(nb, ceil_div(n, int64_t(kScanTile)))) : 1;
  if (b >= nb_real) return;   // uniform for the block
  const int64_t base = int64_t(b) * kScanTile + int64_t(threadIdx.x) * kScanItems;
  int32_t vals[kScanItems];
  int32_t s = 0;
#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    vals[j] = (base + j < n) ? op.value(base + j) : 0;
    s += vals[j];
  }
  __shared__ int32_t tot, prefix;
  int32_t excl = block_exclusive_scan<int32_t>(s, &tot);
  if (threadIdx.x < 32) {
    const int32_t pre = chain_prefix(st, b, tot);
    if (threadIdx.x == 0) {
      prefix = pre;
      if (b == nb_real - 1) op.finish(pre + tot);
    }
  }
  __syncthreads();
  excl += prefix;
#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    if (base + j < n) op.emit(base + j, excl, vals[j]);
    excl += vals[j];
  }
}

struct NewBitsOp {   // words of (new & ~dst): ascending new source ids
  uint32_t* new_bm;
  const uint32_t* dst_bm;
  int64_t n_words;
  const int32_t* n_dst;
  int32_t* src;
  int32_t* pos;
  int32_t* n_src;
  __device__ int64_t size() const { return n_words; }
  __device__ int32_t value(int64_t w) const { return __popc(new_bm[w] & ~dst_bm[w]); }
  __device__ void emit(int64_t w, int32_t excl, int32_t val) const {
    uint32_t word = new_bm[w];
    if (!word) return;
    new_bm[w] = 0u;   // leave the bitmap clean for the next hop
    word &= ~dst_bm[w];
    int32_t idx = *n_dst + excl;
    while (word) {
      const int b = __ffs(word) - 1;
      word &= word - 1;
      const int u = int(w * 32 + b);
      src[idx] = u;
      pos[u] = idx;
      ++idx;
    }
  }
  __device__ void finish(int32_t total) const { *n_src = *n_dst + total; }
};

__global__ void __launch_bounds__(kScanThreads) compact_scan_kernel(NewBitsOp a, uint64_t* stA, int nbA, CntScanOp c,
                                                                    uint64_t* stB, int nbB, int32_t* ticket) {
  APT_PDL_PROLOGUE();
  __shared__ int32_t tk;
  if (threadIdx.x == 0) tk = atomicAdd(ticket, 1);
  __syncthreads();
  const int t = tk;
  if (t < nbA) scan_tile(a, stA, t, nbA);
  else scan_tile(c, stB, t - nbA, nbB);
}

// Exclusive scan of device-counted int32 values (one launch after a tiny reset):
// out[i] = sum_{j<i} cnt[j], out[n] = *total = the sum.
__global__ void scan_reset_kernel(uint64_t* st, int nb, int32_t* ticket) {
  APT_PDL_PROLOGUE();
  for (int i = threadIdx.x; i < nb; i += blockDim.x) st[i] = 0;
  if (threadIdx.x == 0) *ticket = 0;
}

__global__ void __launch_bounds__(kScanThreads) count_scan_kernel(CntScanOp c, uint64_t* st, int nb, int32_t* ticket) {
  APT_PDL_PROLOGUE();
  __shared__ int32_t tk;
  if (threadIdx.x == 0) tk = atomicAdd(ticket, 1);
  __syncthreads();
  scan_tile(c, st, tk, nb);
}

// The same scan when the preceding kernel already zeroed the status words and the
// ticket (ws: nb = scan_tiles(max_n) status pairs, ticket at ws + 2 nb + 2).
int scan_tiles(int64_t max_n) { return int(std::max<int64_t>(1, ceil_div(max_n, kScanTile))); }
cudaError_t launch_scan_counts_prereset(const int32_t* cnt, const int32_t* n_dev, int64_t max_n, int32_t* out,
                                        int32_t* total, int32_t* ws, cudaStream_t st) {
  const int nb = scan_tiles(max_n);
  CntScanOp cop{cnt, n_dev, out, total};
  launch_pdl(count_scan_kernel, dim3(nb), dim3(kScanThreads), 0, st, cop, reinterpret_cast<uint64_t*>(ws), nb,
             ws + 2 * nb + 2);
  return cudaGetLastError();
}

cudaError_t launch_scan_counts(const int32_t* cnt, const int32_t* n_dev, int64_t max_n, int32_t* out, int32_t* total,
                               int32_t* ws, cudaStream_t st) {
  const int nb = int(std::max<int64_t>(1, ceil_div(max_n, kScanTile)));
  uint64_t* status = reinterpret_cast<uint64_t*>(ws);     // ws >= 2*nb + 8 int32
  int32_t* ticket = ws + 2 * nb + 2;
  launch_pdl(scan_reset_kernel, dim3(1), dim3(256), 0, st, status, nb, ticket);
  CntScanOp cop{cnt, n_dev, out, total};
  launch_pdl(count_scan_kernel, dim3(nb), dim3(kScanThreads), 0, st, cop, status, nb, ticket);
  return cudaGetLastError();
}

cudaError_t launch_compact(const CompactArgs& a, cudaStream_t st) {
  const int T = 256;
  const int nbA = int(std::max<int64_t>(1, ceil_div(a.n_words, kScanTile)));
  const int nbB = int(std::max<int64_t>(1, ceil_div(a.max_dst, kScanTile)));
  uint64_t* stA = reinterpret_cast<uint64_t*>(a.partials);            // >= 2*nbA + 8 int32
  int32_t* ticket = a.partials + 2 * nbA + 2;
  uint64_t* stB = reinterpret_cast<uint64_t*>(a.partials2);           // >= 2*nbB + 8 int32
  const int64_t gm = a.grid_cap > 0 ? std::min<int64_t>(a.grid_cap, grid_for(a.max_dst * a.k, T)) : grid_for(a.max_dst * a.k, T);
  launch_pdl(compact_mark_kernel, dim3(gm), dim3(T), 0, st, a.dst, a.n_dst, a.cnt, a.nbr, a.k, a.dst_bm,
                                                                   a.new_bm, a.pos, a.src, stA, nbA, stB, nbB, ticket);
  NewBitsOp bop{a.new_bm, a.dst_bm, a.n_words, a.n_dst, a.src, a.pos, a.n_src};
  CntScanOp cop{a.cnt, a.n_dst, a.indptr, a.n_edges};
  launch_pdl(compact_scan_kernel, dim3(nbA + nbB), dim3(kScanThreads), 0, st, bop, stA, nbA, cop, stB, nbB, ticket);
  launch_pdl(map_indices_kernel, dim3(gm), dim3(T), 0, st, a.dst, a.cnt, a.nbr, a.n_dst, a.k, a.indptr,
                                                                  a.pos, a.indices, a.dst_bm, a.csc_cnt, a.csc_st, a.csc_nb,
                                                                  a.csc_ticket);
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
                                                            int32_t* __restrict__ n_global,
                                                            const int32_t* __restrict__ n_dev) {
  APT_PDL_PROLOGUE();
  if (n_dev) n_train = *n_dev;   // host-batch path: perm holds exactly one global batch
  const int64_t t = n_dev ? 0 : int64_t(*step_ptr % uint64_t(steps_per_epoch));
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
  launch_pdl(select_seeds_kernel, dim3(1), dim3(1024), 0, st, a.perm, a.n_train, a.step, a.steps_per_epoch, a.world, a.rank,
                                          a.batch, a.by_part, a.part, a.seeds, a.n_seeds, a.n_global, a.n_dev);
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
