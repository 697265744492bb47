// agg.cu -- S6+S7: feature gather fused with GraphSAGE mean aggregation, its
// scatter-add backward, and the plain gather / synthetic-feature fill.
//
// z[v] = (1/deg_s(v)) * sum_{e in row v} x[src_e]   (Eq. 1 AGG = mean, P:100, P:261;
// reading O5: fp32 sum, IEEE round-to-nearest division, 0 for an empty row).
//
// B200 design: one warp per destination row.  A row of d features is cut into
// 16-byte vectors (8 bf16 or 4 fp32); when a row has V <= 16 vectors the warp
// splits into G = 32/V lane groups that stream G different edges at once, so a
// warp keeps G*V 16-B loads in flight; the group partials are folded with
// shuffles at the end.  Layer 1 reads the feature store directly by global id
// (no intermediate gathered copy: the gather is fused into the reduction), and
// a row owned by another rank is read through its NVLink peer pointer.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>
#include <cstdlib>

namespace apt {

template <int EPV>
__device__ __forceinline__ void accumulate_vec(float* acc, uint4 raw) {
  if constexpr (EPV == 8) {
    acc_bf16x2(acc[0], acc[1], raw.x); acc_bf16x2(acc[2], acc[3], raw.y);
    acc_bf16x2(acc[4], acc[5], raw.z); acc_bf16x2(acc[6], acc[7], raw.w);
  } else {
    acc[0] += __uint_as_float(raw.x); acc[1] += __uint_as_float(raw.y);
    acc[2] += __uint_as_float(raw.z); acc[3] += __uint_as_float(raw.w);
  }
}

// Edge sources.  row_ptr(u) is the 16-B aligned start of source u's stored row.
struct EllFstoreSrc {            // layer 1: sampler ELL + the feature store (local / peer shards)
  const int32_t* cnt; const int32_t* nbr; int k;
  FeatView fv; int64_t row_bytes;
  __device__ __forceinline__ int64_t begin(int64_t i) const { return i * k; }
  __device__ __forceinline__ int count(int64_t i) const { return cnt[i]; }
  // ids can be read before the count arrives: the ELL row has k slots
  __device__ __forceinline__ int cap(int c) const { return k; }
  __device__ __forceinline__ int node(int64_t e) const { return nbr[e]; }
  __device__ __forceinline__ const char* row_ptr(int u) const {
    if (fv.loc) {   // one 8-byte (tier, row) load: local shard, NVLink peer, host tier or cache
      const int2 l = __ldg(fv.loc + u);
      return reinterpret_cast<const char*>(fv.base[l.x]) + int64_t(l.y) * row_bytes;
    }
    return reinterpret_cast<const char*>(fv.base[0]) + int64_t(u) * row_bytes;
  }
};

struct CsrSrc {                  // upper layers: block CSR over the previous layer's rows (fp32 or bf16)
  const int32_t* indptr; const int32_t* indices; const void* x; int64_t row_bytes;
  __device__ __forceinline__ int64_t begin(int64_t i) const { return indptr[i]; }
  __device__ __forceinline__ int count(int64_t i) const { return indptr[i + 1] - indptr[i]; }
  __device__ __forceinline__ int cap(int c) const { return c; }
  __device__ __forceinline__ int node(int64_t e) const { return indices[e]; }
  __device__ __forceinline__ const char* row_ptr(int u) const {
    return reinterpret_cast<const char*>(x) + int64_t(u) * row_bytes;
  }
};

// Segmented mean with the gather fused in (S6+S7).  A row of V 16-byte vectors
// is owned by a lane group of LG lanes (LG = 16: two destination rows per warp
// when V <= 16; LG = 32 otherwise, VPL = ceil(V/32) vectors per lane).  Per chunk
// of LG edges, every lane resolves ONE edge's row pointer (and, for SNP, its
// partition filter) with coalesced loads; the pointers are then broadcast by
// shuffles and each lane streams its vector of 4 edges at a time (4 independent
// 16-B loads in flight per lane, no dependent index load on the critical path).
// Sum in fp32 (exact under O4), IEEE RN division by the sampled degree (O5).
template <int EPV, int VPL, int LG, class Src>
__global__ void __launch_bounds__(256, (VPL == 1 ? 6 : 4)) agg_kernel(AggArgs a, Src src) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int sub = LG == 16 ? (lane >> 4) : 0;
  const int l = LG == 16 ? (lane & 15) : lane;
  constexpr int RPW = 32 / LG;                                 // destination rows per warp
  const int64_t n_dst = *a.n_dst;
  const int V = int(ceil_div(a.dim, EPV));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; w * RPW < n_dst; w += nwarps) {
    const int64_t i = w * RPW + sub;
    const bool valid = i < n_dst;
    const int cnt = valid ? src.count(i) : 0;
    const int64_t e_base = valid ? src.begin(i) : 0;
    int cmax = cnt;
    if (LG == 16) cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, 16));
    float acc[VPL][EPV];
#pragma unroll
    for (int p = 0; p < VPL; ++p)
#pragma unroll
      for (int q = 0; q < EPV; ++q) acc[p][q] = 0.f;
    constexpr int NB = 4;                                      // 16-B loads in flight per lane (8: more registers, slower)
    for (int e0 = 0; e0 < cmax; e0 += LG) {
      // resolve one edge per lane (ELL: the id load does not wait for the count)
      int u = -1;
      if (valid && e0 + l < src.cap(cnt)) u = src.node(e_base + e0 + l);
      const char* rp = nullptr;
      if (e0 + l < cnt && (!a.filt_part || a.filt_part[u] == a.keep_part)) rp = src.row_ptr(u);
      const int m = min(LG, cmax - e0);
      for (int j = 0; j < m; j += NB) {
        uint4 v[NB][VPL];
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const char* r = reinterpret_cast<const char*>(
              __shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(rp), sub * LG + ((j + q) & (LG - 1))));
          const bool on = (j + q < m) && r != nullptr;
#pragma unroll
          for (int p = 0; p < VPL; ++p) {
            const int jv = l + p * LG;
            v[q][p] = (on && jv < V) ? ld_nc_v4(r + int64_t(jv) * 16) : make_uint4(0, 0, 0, 0);
          }
        }
#pragma unroll
        for (int q = 0; q < NB; ++q)
#pragma unroll
          for (int p = 0; p < VPL; ++p) accumulate_vec<EPV>(acc[p], v[q][p]);
      }
    }
    if (!valid) continue;
    if (a.z_ones && l == 0) {   // 1.0 in column dim: the bias-gradient column of the weight-gradient GEMM
      if (a.z_bf16) a.z_bf16[i * a.z_bf16_pitch + a.dim] = 0x3F80;
      else if (a.z_f32) a.z_f32[i * a.z_f32_pitch + a.dim] = 1.f;
    }
    const float fdeg = float(a.deg_override ? a.deg_override[i] : cnt);
    const float rdeg = fdeg > 0.f ? __frcp_rn(fdeg) : 0.f;   // one reciprocal per row (O5 division below)
#pragma unroll
    for (int p = 0; p < VPL; ++p) {
      const int jv = l + p * LG;
      if (jv >= V) continue;
      float z[EPV];
#pragma unroll
      for (int q = 0; q < EPV; ++q) z[q] = fdeg > 0.f ? div_rn_rcp(acc[p][q], fdeg, rdeg) : 0.f;
      const int c0 = jv * EPV;
      const bool full = c0 + EPV <= a.dim;
      if (a.z_f32) {
        float* o = a.z_f32 + i * a.z_f32_pitch + c0;
        if (full) {
#pragma unroll
          for (int q = 0; q < EPV; q += 4) *reinterpret_cast<float4*>(o + q) = make_float4(z[q], z[q + 1], z[q + 2], z[q + 3]);
        } else {
#pragma unroll
          for (int q = 0; q < EPV; ++q)
            if (c0 + q < a.dim) o[q] = z[q];
        }
      }
      if (a.z_bf16) {
        uint16_t* o = a.z_bf16 + i * a.z_bf16_pitch + c0;
        if (full) {
          if constexpr (EPV == 8) {
            *reinterpret_cast<uint4*>(o) = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]),
                                                      pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
          } else {
            *reinterpret_cast<uint2*>(o) = make_uint2(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]));
          }
        } else {
#pragma unroll
          for (int q = 0; q < EPV; ++q) {
            if (c0 + q < a.dim) {
              __nv_bfloat16 h = __float2bfloat16_rn(z[q]);
              o[q] = *reinterpret_cast<uint16_t*>(&h);
            }
          }
        }
      }
    }
  }
}

// bpsm: grid cap in blocks per SM.  The upper layers' mean uses 4 (A/B: 16 /
// 6 / 4 -> upper forward 50.5 / 50.5 / 49.7 us in the step: room for the sampling branch,
// every warp streams several rows); the layer-1 gather from the store keeps 16.
template <int EPV, class Src>
static cudaError_t dispatch_agg(const AggArgs& a, const Src& s, int bpsm, cudaStream_t st) {
  const int V = int(ceil_div(a.dim, EPV));
  const int threads = 256;
  const int rpw = V <= 16 ? 2 : 1;
  const int64_t blocks = grid_cap(ceil_div(ceil_div(a.max_dst, rpw) * 32, threads), bpsm);
  if (V <= 16) launch_pdl(agg_kernel<EPV, 1, 16, Src>, dim3(blocks), dim3(threads), 0, st, a, s);
  else if (V <= 32) launch_pdl(agg_kernel<EPV, 1, 32, Src>, dim3(blocks), dim3(threads), 0, st, a, s);
  else if (V <= 64) launch_pdl(agg_kernel<EPV, 2, 32, Src>, dim3(blocks), dim3(threads), 0, st, a, s);
  else if (V <= 128) launch_pdl(agg_kernel<EPV, 4, 32, Src>, dim3(blocks), dim3(threads), 0, st, a, s);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

// ----------------------------------------------------- layer 1, branch-free loads
// The layer-1 case (ELL from the sampler, fanout <= 16, rows of <= 16 vectors: two
// destination rows per warp, one edge id per lane) without predicated loads: a lane
// whose edge is padding (past the row's count, or filtered out by SNP) points at a zero
// row in shared memory, so every load of a batch is issued unconditionally through
// generic addressing (feature rows in global / peer / mapped-host memory, the zero row
// in shared memory: no hot spot).  The next row pair's count and edge ids are loaded
// one iteration ahead, so a row pair's critical path starts at its feature-row loads.
template <int EPV, int NB, int MINB>
__global__ void __launch_bounds__(256, MINB) agg_l1_pf_kernel(AggArgs a, EllFstoreSrc src) {
  APT_PDL_PROLOGUE();
  __shared__ uint4 zrow[16];
  if (threadIdx.x < 16) zrow[threadIdx.x] = make_uint4(0, 0, 0, 0);
  __syncthreads();
  const int lane = lane_id();
  const int sub = lane >> 4, l = lane & 15;
  const int64_t n_dst = *a.n_dst;
  const int V = int(ceil_div(a.dim, EPV));
  const int lv = l < V ? l : 0;
  const int k = src.k;
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  int cnt_n = 0, u_n = -1;
  {
    const int64_t i = w * 2 + sub;
    if (i < n_dst) { cnt_n = src.count(i); if (l < k) u_n = src.node(i * k + l); }
  }
  for (; w * 2 < n_dst; w += nwarps) {
    const int64_t i = w * 2 + sub;
    const bool valid = i < n_dst;
    const int cnt = cnt_n, u = u_n;
    {   // next pair's count and ids, consumed one iteration later
      const int64_t i2 = (w + nwarps) * 2 + sub;
      cnt_n = 0; u_n = -1;
      if (i2 < n_dst) { cnt_n = src.count(i2); if (l < k) u_n = src.node(i2 * k + l); }
    }
    const int cmax = max(cnt, __shfl_xor_sync(0xffffffffu, cnt, 16));
    float acc[EPV];
#pragma unroll
    for (int q = 0; q < EPV; ++q) acc[q] = 0.f;
    const bool keep = l < cnt && (!a.filt_part || a.filt_part[u] == a.keep_part);
    const char* rp = keep ? src.row_ptr(u) : reinterpret_cast<const char*>(zrow);
    for (int j = 0; j < cmax; j += NB) {
      uint4 v[NB];
#pragma unroll
      for (int q = 0; q < NB; ++q) {
        const char* r = reinterpret_cast<const char*>(
            __shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(rp), sub * 16 + ((j + q) & 15)));
        // NB not dividing 16: slots past the 16 edge lanes wrap onto real edges, read
        // the zero row instead (cnt <= k <= 16, so every such slot is padding)
        if constexpr ((16 % NB) != 0) if (j + q >= 16) r = reinterpret_cast<const char*>(zrow);
        v[q] = *reinterpret_cast<const uint4*>(r + lv * 16);
      }
#pragma unroll
      for (int q = 0; q < NB; ++q) accumulate_vec<EPV>(acc, v[q]);
    }
    if (!valid || l >= V) continue;
    if (a.z_ones && l == 0) {
      if (a.z_bf16) a.z_bf16[i * a.z_bf16_pitch + a.dim] = 0x3F80;
      else if (a.z_f32) a.z_f32[i * a.z_f32_pitch + a.dim] = 1.f;
    }
    const float fdeg = float(a.deg_override ? a.deg_override[i] : cnt);
    const float rdeg = fdeg > 0.f ? __frcp_rn(fdeg) : 0.f;
    float z[EPV];
#pragma unroll
    for (int q = 0; q < EPV; ++q) z[q] = fdeg > 0.f ? div_rn_rcp(acc[q], fdeg, rdeg) : 0.f;
    const int c0 = l * EPV;
    const bool full = c0 + EPV <= a.dim;
    if (a.z_f32) {
      float* o = a.z_f32 + i * a.z_f32_pitch + c0;
#pragma unroll
      for (int q = 0; q < EPV; ++q)
        if (full || c0 + q < a.dim) o[q] = z[q];
    }
    if (a.z_bf16) {
      uint16_t* o = a.z_bf16 + i * a.z_bf16_pitch + c0;
      if (full) {
        if constexpr (EPV == 8) {
          *reinterpret_cast<uint4*>(o) = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]),
                                                    pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
        } else {
          *reinterpret_cast<uint2*>(o) = make_uint2(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]));
        }
      } else {
#pragma unroll
        for (int q = 0; q < EPV; ++q) {
          if (c0 + q < a.dim) {
            __nv_bfloat16 h = __float2bfloat16_rn(z[q]);
            o[q] = *reinterpret_cast<uint16_t*>(&h);
          }
        }
      }
    }
  }
}

// The same gather for a single-shard view (fv.loc == nullptr: GDP at C = 1, NFP's column
// shard, the benchmark): every row sits in base[0], so a lane broadcasts a 32-bit ROW
// INDEX (padding edges: the shard's zero row fv.zrow) instead of a 64-bit pointer, and an
// edge's load address is one IMAD.WIDE off the lane's column base: per edge and lane one
// shuffle, one address op, one non-coherent 16-B load and 8 mixed-precision adds (the
// pointer form issued two shuffles, two selects and a 64-bit add, and 16 unpack + add
// instructions; ncu had the kernel issue-active 68 % of its cycles).
template <int EPV, int NB, int MINB>
__global__ void __launch_bounds__(256, MINB) agg_l1_flat_kernel(AggArgs a, EllFstoreSrc src) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int sub = lane >> 4, l = lane & 15;
  const int64_t n_dst = *a.n_dst;
  const int V = int(ceil_div(a.dim, EPV));
  const int lv = l < V ? l : 0;
  const int k = src.k;
  // the lane's column base as one opaque 64-bit value, so each edge's address is a single
  // IMAD.WIDE.U32 (row * row_bytes + base) rather than a product plus a separate base add
  uint64_t cbase;
  asm("mov.b64 %0, %1;" : "=l"(cbase) : "l"(reinterpret_cast<uint64_t>(src.fv.base[0]) + uint64_t(lv) * 16u));
  const uint32_t rb = uint32_t(src.row_bytes);
  const int zr = int(src.fv.zrow);
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  int cnt_n = 0, u_n = zr;
  {
    const int64_t i = w * 2 + sub;
    if (i < n_dst) { cnt_n = src.count(i); if (l < k) u_n = src.node(i * k + l); }
  }
  for (; w * 2 < n_dst; w += nwarps) {
    const int64_t i = w * 2 + sub;
    const bool valid = i < n_dst;
    const int cnt = cnt_n, u = u_n;
    {   // next pair's count and ids, consumed one iteration later
      const int64_t i2 = (w + nwarps) * 2 + sub;
      cnt_n = 0; u_n = zr;
      if (i2 < n_dst) { cnt_n = src.count(i2); if (l < k) u_n = src.node(i2 * k + l); }
    }
    const int cmax = max(cnt, __shfl_xor_sync(0xffffffffu, cnt, 16));
    float acc[EPV];
#pragma unroll
    for (int q = 0; q < EPV; ++q) acc[q] = 0.f;
    const bool keep = l < cnt && (!a.filt_part || a.filt_part[u] == a.keep_part);
    const uint32_t ur = uint32_t(keep ? u : zr);
#pragma unroll 1
    for (int j = 0; j < cmax; j += NB) {
      uint4 v[NB];
#pragma unroll
      for (int q = 0; q < NB; ++q) {
        uint32_t uq = __shfl_sync(0xffffffffu, ur, sub * 16 + ((j + q) & 15));
        if constexpr ((16 % NB) != 0) if (j + q >= 16) uq = uint32_t(zr);
        v[q] = __ldg(reinterpret_cast<const uint4*>(cbase + uint64_t(uq) * rb));   // L1-allocating: the zero row stays in L1
      }
#pragma unroll
      for (int q = 0; q < NB; ++q) accumulate_vec<EPV>(acc, v[q]);
    }
    if (!valid || l >= V) continue;
    if (a.z_ones && l == 0) {
      if (a.z_bf16) a.z_bf16[i * a.z_bf16_pitch + a.dim] = 0x3F80;
      else if (a.z_f32) a.z_f32[i * a.z_f32_pitch + a.dim] = 1.f;
    }
    const float fdeg = float(a.deg_override ? a.deg_override[i] : cnt);
    const float rdeg = fdeg > 0.f ? __frcp_rn(fdeg) : 0.f;
    float z[EPV];
#pragma unroll
    for (int q = 0; q < EPV; ++q) z[q] = fdeg > 0.f ? div_rn_rcp(acc[q], fdeg, rdeg) : 0.f;
    const int c0 = l * EPV;
    const bool full = c0 + EPV <= a.dim;
    if (a.z_f32) {
      float* o = a.z_f32 + i * a.z_f32_pitch + c0;
#pragma unroll
      for (int q = 0; q < EPV; ++q)
        if (full || c0 + q < a.dim) o[q] = z[q];
    }
    if (a.z_bf16) {
      uint16_t* o = a.z_bf16 + i * a.z_bf16_pitch + c0;
      if (full) {
        if constexpr (EPV == 8) {
          *reinterpret_cast<uint4*>(o) = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]),
                                                    pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
        } else {
          *reinterpret_cast<uint2*>(o) = make_uint2(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]));
        }
      } else {
#pragma unroll
        for (int q = 0; q < EPV; ++q) {
          if (c0 + q < a.dim) {
            __nv_bfloat16 h = __float2bfloat16_rn(z[q]);
            o[q] = *reinterpret_cast<uint16_t*>(&h);
          }
        }
      }
    }
  }
}

cudaError_t launch_agg_fstore(const AggArgs& a, const FeatView& fv, cudaStream_t st) {
  EllFstoreSrc s{a.cnt, a.nbr, a.k, fv, fv.pitch * (fv.dtype == kBF16 ? 2 : 4)};
  AggArgs b = a;
  b.dim = fv.dim;
  const int epv = fv.dtype == kBF16 ? 8 : 4;
  const int V = int(ceil_div(b.dim, epv));
  // NB 5 loads in flight per lane (a fanout-10 row in two rounds) at 64 registers, the
  // grid one resident wave: every warp streams several row pairs, so the one-ahead index
  // prefetch pays and there is no partial last wave (A/B in DESIGN §8: 30.2 us in the
  // step vs 32.4 at 16 blocks per SM and 33.2-34.5 for NB 4 / 8 and 48 registers)
  static const int flat_ok = [] { const char* v = std::getenv("APT_AGG_FLAT"); return v ? atoi(v) : 1; }();
  if (V <= 16 && b.k <= 16 && !fv.loc && fv.zrow >= 0 && flat_ok) {
    if (fv.dtype == kBF16) {
      // 10 loads in flight per lane (a fanout-10 row in one round) at 3 blocks per SM (75
      // registers): A/B in the step 27.8 vs 28.9 us for 5 loads at 4 blocks per SM; 10 at 4
      // (spills) 34.0, 5 at 5 29.5, 4 at 5 29.6 (APT_FLAT_VAR 1-4)
      static const int var = [] { const char* v = std::getenv("APT_FLAT_VAR"); return v ? atoi(v) : 2; }();
      auto kern = var == 1 ? agg_l1_flat_kernel<8, 10, 4> : var == 0 ? agg_l1_flat_kernel<8, 5, 4>
                : var == 3 ? agg_l1_flat_kernel<8, 5, 5> : var == 4 ? agg_l1_flat_kernel<8, 4, 5>
                : agg_l1_flat_kernel<8, 10, 3>;
      const int64_t blocks = grid_cap(ceil_div(ceil_div(b.max_dst, 2) * 32, 256),
                                      b.bpsm > 0 ? b.bpsm : resident_blocks(kern, 256));
      launch_pdl(kern, dim3(blocks), dim3(256), 0, st, b, s);
    } else {
      auto kern = agg_l1_flat_kernel<4, 4, 6>;
      const int64_t blocks = grid_cap(ceil_div(ceil_div(b.max_dst, 2) * 32, 256),
                                      b.bpsm > 0 ? b.bpsm : resident_blocks(kern, 256));
      launch_pdl(kern, dim3(blocks), dim3(256), 0, st, b, s);
    }
    return cudaGetLastError();
  }
  if (V <= 16 && b.k <= 16) {
    if (fv.dtype == kBF16) {
      auto kern = agg_l1_pf_kernel<8, 5, 4>;
      const int64_t blocks = grid_cap(ceil_div(ceil_div(b.max_dst, 2) * 32, 256),
                                      b.bpsm > 0 ? b.bpsm : resident_blocks(kern, 256));
      launch_pdl(kern, dim3(blocks), dim3(256), 0, st, b, s);
    } else {
      auto kern = agg_l1_pf_kernel<4, 4, 6>;
      const int64_t blocks = grid_cap(ceil_div(ceil_div(b.max_dst, 2) * 32, 256),
                                      b.bpsm > 0 ? b.bpsm : resident_blocks(kern, 256));
      launch_pdl(kern, dim3(blocks), dim3(256), 0, st, b, s);
    }
    return cudaGetLastError();
  }
  return fv.dtype == kBF16 ? dispatch_agg<8>(b, s, 16, st) : dispatch_agg<4>(b, s, 16, st);
}

// Upper-layer mean over bf16 rows of 17..32 16-byte vectors (d' in (128, 256]; reading
// R11): agg_kernel<8, 1, 32, CsrSrc>'s warp-per-row form with the flat gather's
// addressing -- the edge's source row broadcast as a 32-bit index, one IMAD.WIDE off the
// lane's opaque column base, unconditional loads of always-valid rows (lanes past the
// row's count hold row 0), padding zeroed by selects.  Same edge order, same adds, same
// division and rounding: Z is bit-identical to agg_kernel's.
template <int NB, int MINB>   // source rows in flight per warp, blocks per SM
__global__ void __launch_bounds__(256, MINB) agg_csr_b8_kernel(AggArgs a, uint32_t rb) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n_dst = *a.n_dst;
  const int V = int(ceil_div(a.dim, 8));
  const int lv = lane < V ? lane : 0;
  uint64_t base;
  asm("mov.b64 %0, %1;" : "=l"(base) : "l"(reinterpret_cast<uint64_t>(a.xb) + uint64_t(lv) * 16u));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n_dst; i += nwarps) {
    const int e0 = a.indptr[i];
    const int cnt = a.indptr[i + 1] - e0;
    float acc[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
    for (int c0 = 0; c0 < cnt; c0 += 32) {
      const uint32_t u = c0 + lane < cnt ? uint32_t(a.indices[e0 + c0 + lane]) : 0u;
      const int m = min(32, cnt - c0);
#pragma unroll 1
      for (int j = 0; j < m; j += NB) {
        uint4 v[NB];
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const uint32_t uq = __shfl_sync(0xffffffffu, u, (j + q) & 31);
          const uint4 t = __ldg(reinterpret_cast<const uint4*>(base + uint64_t(uq) * rb));
          v[q] = j + q < m ? t : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int q = 0; q < NB; ++q) accumulate_vec<8>(acc, v[q]);
      }
    }
    if (a.z_ones && lane == 0) a.z_bf16[i * a.z_bf16_pitch + a.dim] = 0x3F80;
    if (lane >= V) continue;
    const float fdeg = float(cnt);
    const float rdeg = fdeg > 0.f ? __frcp_rn(fdeg) : 0.f;
    float z[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) z[q] = fdeg > 0.f ? div_rn_rcp(acc[q], fdeg, rdeg) : 0.f;
    const int c0 = lane * 8;
    uint16_t* o = a.z_bf16 + i * a.z_bf16_pitch + c0;
    if (c0 + 8 <= a.dim) {
      *reinterpret_cast<uint4*>(o) = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]),
                                                pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
    } else {
#pragma unroll
      for (int q = 0; q < 8; ++q)
        if (c0 + q < a.dim) o[q] = bf16_bits(z[q]);
    }
  }
}

cudaError_t launch_agg_csr(const AggArgs& a, cudaStream_t st) {
  // rows wider than one launch covers (> 128 16-B vectors): column chunks of 512 fp32 /
  // 1024 bf16 columns
  const bool bf = a.xb != nullptr;
  const int kChunk = bf ? 1024 : 512;
  for (int c0 = 0; c0 < a.dim; c0 += kChunk) {
    AggArgs b = a;
    b.dim = std::min(kChunk, a.dim - c0);
    if (a.z_f32) b.z_f32 = a.z_f32 + c0;
    if (a.z_bf16) b.z_bf16 = a.z_bf16 + c0;
    b.z_ones = (c0 + b.dim == a.dim) ? a.z_ones : 0;   // column a.dim, written by the last chunk
    cudaError_t e;
    static const int csr_flat = [] { const char* v = std::getenv("APT_AGG_CSR_FLAT"); return v ? atoi(v) : 1; }();
    const int Vb = int(ceil_div(b.dim, 8));
    if (bf && csr_flat && Vb > 16 && Vb <= 32 && !b.deg_override && !b.filt_part && b.z_bf16 && !b.z_f32 &&
        (a.x_pitch * 2) % 16 == 0 && (reinterpret_cast<uintptr_t>(a.xb) & 15) == 0) {
      b.xb = a.xb + c0;
      // APT_CSR_NB: rows in flight per warp (4 at 4 blocks/SM, 6 at 4, 8 at 3; A/B)
      static const int nb = [] { const char* v = std::getenv("APT_CSR_NB"); return v ? atoi(v) : 4; }();
      auto kern = nb >= 8 ? agg_csr_b8_kernel<8, 3> : nb >= 6 ? agg_csr_b8_kernel<6, 4> : agg_csr_b8_kernel<4, 4>;
      const int64_t blocks = grid_cap(ceil_div(b.max_dst * 32, 256), nb >= 8 ? 3 : 4);
      launch_pdl(kern, dim3(blocks), dim3(256), 0, st, b, uint32_t(a.x_pitch * 2));
      e = cudaGetLastError();
    } else if (bf) {
      CsrSrc s{b.indptr, b.indices, a.xb + c0, a.x_pitch * 2};
      e = dispatch_agg<8>(b, s, 4, st);
    } else {
      CsrSrc s{b.indptr, b.indices, a.x + c0, a.x_pitch * 4};
      e = dispatch_agg<4>(b, s, 4, st);
    }
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// ---------------------------------------------------------------- backward
// dX[src_e] += dZ[v] / deg_s(v): one warp per dst, the dZ row held in registers,
// one 16-B vector red per lane per edge.
__global__ void __launch_bounds__(256) agg_bwd_kernel(const int32_t* __restrict__ indptr,
                                                      const int32_t* __restrict__ indices,
                                                      const int32_t* __restrict__ n_dst_p, const float* __restrict__ dz,
                                                      int64_t dz_pitch, int dim, float* __restrict__ dx,
                                                      int64_t dx_pitch) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n_dst = *n_dst_p;
  const int V = int(ceil_div(dim, 4));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n_dst; i += nwarps) {
    const int e0 = indptr[i], e1 = indptr[i + 1];
    if (e1 == e0) continue;
    const float fdeg = float(e1 - e0);
    for (int j = lane; j < V; j += 32) {
      const float4 g = *reinterpret_cast<const float4*>(dz + i * dz_pitch + j * 4);
      const float a = div_rn(g.x, fdeg), b = div_rn(g.y, fdeg), c = div_rn(g.z, fdeg), d = div_rn(g.w, fdeg);
      for (int e = e0; e < e1; ++e) red_add_v4(dx + int64_t(indices[e]) * dx_pitch + j * 4, a, b, c, d);
    }
  }
}

cudaError_t launch_agg_bwd(const int32_t* indptr, const int32_t* indices, const int32_t* n_dst, int64_t max_dst,
                           const float* dz, int64_t dz_pitch, int dim, float* dx, int64_t dx_pitch, cudaStream_t st) {
  int64_t blocks = grid_cap(ceil_div(max_dst * 32, 256), 16);
  launch_pdl(agg_bwd_kernel, dim3(blocks), dim3(256), 0, st, indptr, indices, n_dst, dz, dz_pitch, dim, dx, dx_pitch);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- gather
__global__ void gather_kernel(FeatView fv, const int32_t* __restrict__ ids, const int32_t* __restrict__ n_p,
                              int64_t n_static, char* __restrict__ out, int64_t out_pitch_bytes) {
  APT_PDL_PROLOGUE();
  const int64_t n = n_p ? int64_t(*n_p) : n_static;
  const int esz = fv.dtype == kBF16 ? 2 : 4;
  const int V = int(ceil_div(int64_t(fv.dim) * esz, 16));
  const int lane = lane_id();
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n; i += nwarps) {
    const int u = ids[i];
    const int2 l = fv.loc ? __ldg(fv.loc + u) : make_int2(0, u);
    const char* row = fv.loc ? reinterpret_cast<const char*>(fv.base[l.x]) + int64_t(l.y) * fv.pitch * esz
                              : reinterpret_cast<const char*>(fv.base[0]) + int64_t(u) * fv.pitch * esz;
    for (int j = lane; j < V; j += 32)
      *reinterpret_cast<uint4*>(out + i * out_pitch_bytes + j * 16) = ld_nc_v4(row + j * 16);
  }
}

cudaError_t launch_gather(const FeatView& fv, const int32_t* ids, const int32_t* n_dev, int64_t max_n, void* out,
                          int64_t out_pitch, cudaStream_t st) {
  int64_t blocks = grid_cap(ceil_div(max_n * 32, 256), 16);
  const int esz = fv.dtype == kBF16 ? 2 : 4;
  launch_pdl(gather_kernel, dim3(blocks), dim3(256), 0, st, fv, ids, n_dev, max_n, reinterpret_cast<char*>(out), out_pitch * esz);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- features
__global__ void fill_features_kernel(void* shard, int bf16, int64_t pitch, int col0, int ncols,
                                     const int32_t* __restrict__ ids, int64_t n, uint2 key) {
  const int64_t total = n * pitch;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / pitch;
    const int c = int(t - r * pitch);
    const float v = c < ncols ? feature_value(key, ids ? ids[r] : r, col0 + c) : 0.f;
    if (bf16) {
      __nv_bfloat16 h = __float2bfloat16_rn(v);
      reinterpret_cast<uint16_t*>(shard)[t] = *reinterpret_cast<uint16_t*>(&h);
    } else {
      reinterpret_cast<float*>(shard)[t] = v;
    }
  }
}

cudaError_t launch_fill_features(void* shard, DType dt, int64_t pitch, int col0, int ncols, const int32_t* ids,
                                 int64_t n, uint64_t seed, cudaStream_t st) {
  int64_t blocks = grid_cap(ceil_div(n * pitch, 256), 64);
  fill_features_kernel<<<blocks, 256, 0, st>>>(shard, dt == kBF16, pitch, col0, ncols, ids, n,
                                               philox_key(seed, kDomFeat));
  return cudaGetLastError();
}

}  // namespace apt

// ---------------------------------------------------------------- self-test
// Exhaustive check of div_rn_rcp against the IEEE division for every mean the
// method can form under O4 (x = m/64, |m| <= 2^17, d = 1..256) plus random
// normal floats: counts bitwise mismatches.
namespace apt {
__global__ void selftest_div_kernel(unsigned long long* bad) {
  const int64_t total = (int64_t(1) << 18) * 256;
  unsigned long long nb = 0;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int d = int(t & 255) + 1;
    const int m = int(t >> 8) - (1 << 17);
    const float x = float(m) * (1.0f / 64.0f);
    const float fd = float(d);
    const float a = div_rn_rcp(x, fd, __frcp_rn(fd)), b = __fdiv_rn(x, fd);
    if (__float_as_uint(a) != __float_as_uint(b) && !(a == 0.f && b == 0.f)) ++nb;
    // random normal numerator (hash of t), same denominators
    uint32_t h = uint32_t(t) * 2654435761u ^ 0x9E3779B9u;
    h ^= h >> 15; h *= 0x85EBCA6Bu; h ^= h >> 13;
    const float y = __uint_as_float((h & 0x807FFFFFu) | (uint32_t(100 + (h >> 24) % 60) << 23));
    const float c = div_rn_rcp(y, fd, __frcp_rn(fd)), e = __fdiv_rn(y, fd);
    if (__float_as_uint(c) != __float_as_uint(e)) ++nb;
  }
  if (nb) atomicAdd(bad, nb);
}
}  // namespace apt

extern "C" int64_t apt_selftest_div(void) {
  unsigned long long* d = nullptr;
  if (cudaMalloc(&d, 8) != cudaSuccess) return -1;
  cudaMemset(d, 0, 8);
  apt::selftest_div_kernel<<<apt::num_sms() * 8, 256>>>(d);
  unsigned long long h = 0;
  if (cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost) != cudaSuccess) h = ~0ull;
  cudaFree(d);
  return int64_t(h);
}
