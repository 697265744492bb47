// sort.cu -- S1: the epoch permutation's sort (reading O1: perm = train ascending by
// (Philox key, id), "an epoch covers all seeds" in a random order).
//
// A stable least-significant-digit radix sort of (uint64 key, int32 id) pairs, 8 passes
// of 8 bits.  The input ids arrive ascending, so stability orders equal keys by id --
// exactly O1's tie rule.  Per pass three launches:
//   hist    : every 2048-item tile counts its digits (shared-memory atomics) and writes
//             them digit-major, hist[d * nb + b], so that
//   scan    : one exclusive scan of the flat histogram gives every (digit, tile) its
//             output offset (all smaller digits, then the same digit of earlier tiles);
//   scatter : every tile ranks its items stably -- warp w owns items [256w, 256w + 256),
//             rounds of 32 in order, __match_any_sync groups a round's equal digits, a
//             per-warp running count per digit gives the rank, a prefix over the warps
//             orders the warps -- and writes each pair to offset + rank.
// Runs once per epoch (set_epoch), off the step path; n <= 2^31.
#include "common.cuh"
#include "kernels.h"

namespace apt {

namespace {
constexpr int kThreads = 256, kIpt = 8, kTile = kThreads * kIpt, kWarps = kThreads / 32;

__global__ void radix_hist_kernel(const uint64_t* __restrict__ keys, int64_t n, int shift, int nb,
                                  uint32_t* __restrict__ hist) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const int64_t base = int64_t(blockIdx.x) * kTile;
  for (int j = threadIdx.x; j < kTile; j += kThreads) {
    const int64_t i = base + j;
    if (i < n) atomicAdd(&h[uint32_t(keys[i] >> shift) & 255u], 1u);
  }
  __syncthreads();
  hist[int64_t(threadIdx.x) * nb + blockIdx.x] = h[threadIdx.x];
}

// Exclusive scan of hist[0, len) in place, one block of 1024 threads, chunks of 4096.
__global__ void radix_scan_kernel(uint32_t* __restrict__ hist, int64_t len) {
  __shared__ uint32_t wsum[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t c0 = 0; c0 < len; c0 += 4096) {
    uint32_t v[4], s = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t i = c0 + int64_t(threadIdx.x) * 4 + q;
      v[q] = i < len ? hist[i] : 0u;
      s += v[q];
    }
    uint32_t x = s;   // inclusive warp scan of the per-thread sums
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[w] = x;
    __syncthreads();
    if (w == 0) {
      uint32_t t = wsum[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
        if (lane >= o) t += y;
      }
      wsum[lane] = t;   // inclusive over warps
    }
    __syncthreads();
    uint32_t run = carry + (w ? wsum[w - 1] : 0u) + (x - s);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t i = c0 + int64_t(threadIdx.x) * 4 + q;
      if (i < len) hist[i] = run;
      run += v[q];
    }
    __syncthreads();
    if (threadIdx.x == 0) carry += wsum[31];
    __syncthreads();
  }
}

__global__ void radix_scatter_kernel(const uint64_t* __restrict__ kin, const int32_t* __restrict__ vin, int64_t n,
                                     int shift, int nb, const uint32_t* __restrict__ off,
                                     uint64_t* __restrict__ kout, int32_t* __restrict__ vout) {
  __shared__ uint32_t cnt[kWarps][256];
  for (int d = threadIdx.x; d < kWarps * 256; d += kThreads) (&cnt[0][0])[d] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const int64_t base = int64_t(blockIdx.x) * kTile + int64_t(w) * (kIpt * 32);
  uint64_t k[kIpt];
  int32_t v[kIpt];
  uint32_t rank[kIpt];
#pragma unroll
  for (int r = 0; r < kIpt; ++r) {
    const int64_t i = base + r * 32 + lane;
    const bool ok = i < n;
    k[r] = ok ? kin[i] : 0ull;
    v[r] = ok ? vin[i] : 0;
    const uint32_t active = __ballot_sync(0xffffffffu, ok);
    rank[r] = 0;
    if (ok) {
      const uint32_t d = uint32_t(k[r] >> shift) & 255u;
      const uint32_t peers = __match_any_sync(active, d);
      rank[r] = cnt[w][d] + __popc(peers & lt);
      __syncwarp(active);
      if ((peers & lt) == 0) cnt[w][d] += __popc(peers);   // the group's lowest lane
    }
    __syncwarp();
  }
  __syncthreads();
  {   // exclusive prefix over the warps, per digit (thread = digit)
    const int d = threadIdx.x;
    uint32_t run = 0;
#pragma unroll
    for (int q = 0; q < kWarps; ++q) {
      const uint32_t t = cnt[q][d];
      cnt[q][d] = run;
      run += t;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kIpt; ++r) {
    const int64_t i = base + r * 32 + lane;
    if (i >= n) continue;
    const uint32_t d = uint32_t(k[r] >> shift) & 255u;
    const int64_t o = int64_t(off[int64_t(d) * nb + blockIdx.x]) + cnt[w][d] + rank[r];
    kout[o] = k[r];
    vout[o] = v[r];
  }
}
}  // namespace

size_t radix_sort_pairs_scratch(int64_t n) {
  const int64_t nb = ceil_div(std::max<int64_t>(n, 1), kTile);
  return size_t(n) * (sizeof(uint64_t) + sizeof(int32_t)) + size_t(nb) * 256 * sizeof(uint32_t) + 256;
}

// Sorts (keys, vals)[0, n) in place by key, stably; scratch: radix_sort_pairs_scratch(n) bytes.
cudaError_t launch_radix_sort_pairs(uint64_t* keys, int32_t* vals, int64_t n, void* scratch, cudaStream_t st) {
  if (n <= 1) return cudaSuccess;
  if (n > (int64_t(1) << 31)) return cudaErrorInvalidValue;
  const int nb = int(ceil_div(n, kTile));
  uint8_t* s = static_cast<uint8_t*>(scratch);
  uint64_t* k2 = reinterpret_cast<uint64_t*>(s);
  int32_t* v2 = reinterpret_cast<int32_t*>(s + size_t(n) * sizeof(uint64_t));
  uint32_t* hist = reinterpret_cast<uint32_t*>(
      s + round_up(int64_t(n) * (sizeof(uint64_t) + sizeof(int32_t)), 256));
  uint64_t* ka = keys;
  int32_t* va = vals;
  for (int shift = 0; shift < 64; shift += 8) {   // 8 passes: the result lands back in (keys, vals)
    radix_hist_kernel<<<nb, kThreads, 0, st>>>(ka, n, shift, nb, hist);
    radix_scan_kernel<<<1, 1024, 0, st>>>(hist, int64_t(nb) * 256);
    radix_scatter_kernel<<<nb, kThreads, 0, st>>>(ka, va, n, shift, nb, hist, ka == keys ? k2 : keys,
                                                  ka == keys ? v2 : vals);
    ka = ka == keys ? k2 : keys;
    va = va == vals ? v2 : vals;
  }
  return cudaGetLastError();
}

}  // namespace apt

#include <algorithm>
#include <numeric>
#include <vector>

// Self-test of the radix sort's stability (apt.h): n pairs with keys drawn from Philox
// and masked to `key_bits` bits (many equal keys), values 0..n-1; the number of
// positions where the device result differs from std::stable_sort on the host, or < 0
// on a CUDA failure.  Uses the current device.
extern "C" int64_t apt_selftest_sort(int64_t n, uint64_t seed, int key_bits) {
  using namespace apt;
  if (n < 1 || key_bits < 1 || key_bits > 64) return -1;
  std::vector<uint64_t> k(n);
  std::vector<int32_t> v(n);
  const uint2 key = philox_key(seed, kDomPerm);
  const uint64_t mask = key_bits == 64 ? ~0ull : ((1ull << key_bits) - 1);
  for (int64_t i = 0; i < n; ++i) {
    const uint4 w = philox(make_uint4(uint32_t(i), uint32_t(uint64_t(i) >> 32), 0xABCu, 0u), key);
    k[i] = (uint64_t(w.x) | (uint64_t(w.y) << 32)) & mask;
    v[i] = int32_t(i);
  }
  uint64_t* dk = nullptr;
  int32_t* dv = nullptr;
  void* scratch = nullptr;
  if (cudaMalloc(&dk, n * 8) != cudaSuccess || cudaMalloc(&dv, n * 4) != cudaSuccess ||
      cudaMalloc(&scratch, radix_sort_pairs_scratch(n)) != cudaSuccess)
    return -2;
  cudaMemcpy(dk, k.data(), n * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dv, v.data(), n * 4, cudaMemcpyHostToDevice);
  cudaError_t e = launch_radix_sort_pairs(dk, dv, n, scratch, 0);
  std::vector<uint64_t> gk(n);
  std::vector<int32_t> gv(n);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaMemcpy(gk.data(), dk, n * 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(gv.data(), dv, n * 4, cudaMemcpyDeviceToHost);
  cudaFree(dk);
  cudaFree(dv);
  cudaFree(scratch);
  if (e != cudaSuccess) return -3;
  std::vector<int32_t> idx(n);
  std::iota(idx.begin(), idx.end(), 0);
  std::stable_sort(idx.begin(), idx.end(), [&](int32_t a, int32_t b) { return k[a] < k[b]; });
  int64_t bad = 0;
  for (int64_t i = 0; i < n; ++i) bad += (gv[i] != idx[i] || gk[i] != k[idx[i]]) ? 1 : 0;
  return bad;
}
