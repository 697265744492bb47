// bwd.cu -- the mean's backward as a gather (S10): G_{l-1} = relu'(H_{l-1}) * D^T (dZ_l / deg).
//
// The scatter form (dX[src_e] += dZ[v]/deg(v), agg_bwd_kernel) needs a zeroed fp32
// buffer, ~E red.v4 atomics and a separate masking/bf16 pass.  Here the sampled
// block is transposed once per step (counting sort: count, scan, fill -- built on
// the side stream while the forward runs) and every source row pulls its in-edges:
// one pass reads dZ (L2-resident), the ReLU mask from H, and writes G (fp32) and/or
// its bf16 copy directly; no atomics, no zeroing.  Within a row the in-edges are
// summed in their CSC order, which the fill's atomic slot counters make
// scheduling-dependent: G is not bitwise reproducible run to run (fp32 sums of the same
// terms in another order; the parity tests' T1 allowance covers it).
#include "common.cuh"
#include "kernels.h"
#include <algorithm>

namespace apt {

cudaError_t launch_scan_counts(const int32_t* cnt, const int32_t* n_dev, int64_t max_n, int32_t* out, int32_t* total,
                               int32_t* ws, cudaStream_t st);
int scan_tiles(int64_t max_n);
cudaError_t launch_scan_counts_prereset(const int32_t* cnt, const int32_t* n_dev, int64_t max_n, int32_t* out,
                                        int32_t* total, int32_t* ws, cudaStream_t st);

// in-degree of every local source of the block; also zeroes the next scan's status
// words and ticket (one launch fewer on the sampling branch)
__global__ void csc_count_kernel(const int32_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                 const int32_t* __restrict__ n_edges_p, int32_t* __restrict__ cnt,
                                 uint64_t* __restrict__ scan_st, int scan_nb, int32_t* __restrict__ scan_ticket) {
  APT_PDL_PROLOGUE();
  if (scan_st) {
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i <= scan_nb; i += int64_t(gridDim.x) * blockDim.x) {
      if (i < scan_nb) scan_st[i] = 0;
      else *scan_ticket = 0;
    }
  }
  const int64_t E = *n_edges_p;
  for (int64_t e = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < E; e += int64_t(gridDim.x) * blockDim.x)
    atomicAdd(cnt + indices[e], 1);
}

// csc_dst[csc_ptr[u] + j] = (v, deg(v)) for the j-th in-edge (v, u): the pull reads the
// destination and its sampled degree with one 8-B load.  Counts return to 0 (ready for
// the next step).
__global__ void csc_fill_kernel(const int32_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                const int32_t* __restrict__ n_dst_p, const int32_t* __restrict__ csc_ptr,
                                int32_t* __restrict__ cnt, int2* __restrict__ csc_dst) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_dst_p;
  for (int64_t v = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; v < n; v += int64_t(gridDim.x) * blockDim.x) {
    const int b = indptr[v], e1 = indptr[v + 1];
    for (int e = b; e < e1; ++e) {
      const int u = indices[e];
      csc_dst[csc_ptr[u] + atomicSub(cnt + u, 1) - 1] = make_int2(int32_t(v), e1 - b);
    }
  }
}

// The same fill with one thread per (row, slot) of the sampler's fixed fanout k: no
// per-row loop of dependent atomics (A/B: APT_CSC_SLOTS=0 keeps the row loop).  Either
// fill orders a row's in-edges by the order its atomicSub calls land.
__global__ void csc_fill_slots_kernel(const int32_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                      const int32_t* __restrict__ n_dst_p, int k, const int32_t* __restrict__ csc_ptr,
                                      int32_t* __restrict__ cnt, int2* __restrict__ csc_dst) {
  APT_PDL_PROLOGUE();
  const int64_t slots = int64_t(*n_dst_p) * k;
  for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < slots; s += int64_t(gridDim.x) * blockDim.x) {
    const int64_t v = s / k;
    const int q = int(s - v * k);
    const int b = indptr[v], deg = indptr[v + 1] - b;
    if (q >= deg) continue;
    const int u = indices[b + q];
    csc_dst[csc_ptr[u] + atomicSub(cnt + u, 1) - 1] = make_int2(int32_t(v), deg);
  }
}

cudaError_t launch_csc_build(const CscArgs& a, cudaStream_t st) {
  const int64_t T = 256;
  const int64_t cap = a.grid_cap > 0 ? a.grid_cap : int64_t(num_sms()) * 16;
  const int64_t ge = std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.max_edges, T), cap));
  const int nb = scan_tiles(a.max_src);
  if (!a.counted)
    launch_pdl(csc_count_kernel, dim3(ge), dim3(T), 0, st, a.indptr, a.indices, a.n_edges, a.cnt,
               reinterpret_cast<uint64_t*>(a.ws), nb, a.ws + 2 * nb + 2);
  cudaError_t e = launch_scan_counts_prereset(a.cnt, a.n_src, a.max_src, a.csc_ptr, a.csc_total, a.ws, st);
  if (e != cudaSuccess) return e;
  static const int slots = [] { const char* v = std::getenv("APT_CSC_SLOTS"); return v ? atoi(v) : 1; }();
  if (slots && a.k > 0) {
    const int64_t gs = std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.max_dst * a.k, T), cap));
    launch_pdl(csc_fill_slots_kernel, dim3(gs), dim3(T), 0, st, a.indptr, a.indices, a.n_dst, a.k, a.csc_ptr, a.cnt,
               a.csc_dst);
    return cudaGetLastError();
  }
  const int64_t gd = std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.max_dst, T), cap));
  launch_pdl(csc_fill_kernel, dim3(gd), dim3(T), 0, st, a.indptr, a.indices, a.n_dst, a.csc_ptr, a.cnt, a.csc_dst);
  return cudaGetLastError();
}

// One warp per R source rows u (VPL float4 vectors per lane per row): g = sum over
// in-edges of dZ[v] / deg(v) (correctly rounded per term, reading O5), masked by
// H[u] > 0.  Latency design (the layer-1 pull has ~1 in-edge per row, so the kernel is
// a chain of dependent loads, not a stream): the R rows of a warp are in flight at
// once; each row's ReLU mask is loaded with its CSC bounds (independent of the edge
// chain); the in-edges' (v, deg) pairs come with one coalesced 8-B load per lane and
// are broadcast by shuffles, so a row costs three dependent loads (bounds -> edges ->
// dZ rows) instead of five.
// MS = mask source: 0 none, 1 bit mask, 2 fp32 H, 3 bf16 H.  The raw mask words are
// loaded with the CSC bounds and decoded only after the edge loop (a DRAM-latency H
// read overlaps the bounds -> edges -> dZ chain instead of stalling it).
template <int MS> struct MaskRaw { uint32_t w; };
template <> struct MaskRaw<2> { float4 w; };
template <> struct MaskRaw<3> { uint2 w; };

template <int MS>
__device__ __forceinline__ MaskRaw<MS> load_mask(const PullArgs& a, int64_t u, int j) {
  MaskRaw<MS> m;
  if constexpr (MS == 0) m.w = 0xFu;
  if constexpr (MS == 1) m.w = uint32_t(a.mask[u * a.mask_pitch + (j * 4) / 16]) >> ((j * 4) & 15);
  if constexpr (MS == 2) m.w = __ldg(reinterpret_cast<const float4*>(a.h + u * a.h_pitch + j * 4));
  if constexpr (MS == 3) m.w = __ldg(reinterpret_cast<const uint2*>(a.hb + u * a.hb_pitch + j * 4));
  return m;
}
__device__ __forceinline__ uint32_t bf16_pos(uint32_t h16) { return (h16 != 0u && !(h16 & 0x8000u)) ? 1u : 0u; }
template <int MS>
__device__ __forceinline__ uint32_t decode_mask(const MaskRaw<MS>& m) {
  if constexpr (MS == 0 || MS == 1) return m.w & 0xFu;
  if constexpr (MS == 2)
    return (m.w.x > 0.f ? 1u : 0u) | (m.w.y > 0.f ? 2u : 0u) | (m.w.z > 0.f ? 4u : 0u) | (m.w.w > 0.f ? 8u : 0u);
  if constexpr (MS == 3)
    return bf16_pos(m.w.x & 0xFFFFu) | (bf16_pos(m.w.x >> 16) << 1) | (bf16_pos(m.w.y & 0xFFFFu) << 2) |
           (bf16_pos(m.w.y >> 16) << 3);
  return 0xFu;
}

template <int VPL, int R, int MS>
__global__ void __launch_bounds__(256) pull_bwd_kernel(PullArgs a) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n = *a.n_src;
  const int V = int(ceil_div(a.dim, 4));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  const int64_t rows_out = a.gb ? std::min<int64_t>(a.max_src, round_up(n, 64)) : n;
  for (int64_t u0 = ((int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5) * R; u0 < rows_out; u0 += nwarps * R) {
    int e0[R], cnt[R];
    MaskRaw<MS> mraw[R][VPL];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r;
      e0[r] = 0; cnt[r] = 0;
      if (u < n) { e0[r] = a.csc_ptr[u]; cnt[r] = a.csc_ptr[u + 1] - e0[r]; }
#pragma unroll
      for (int p = 0; p < VPL; ++p) {
        const int j = lane + 32 * p;
        if (u < n && j < V) mraw[r][p] = load_mask<MS>(a, u, j);
        else mraw[r][p] = MaskRaw<MS>{};
      }
    }
    float acc[R][VPL][4];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int p = 0; p < VPL; ++p) acc[r][p][0] = acc[r][p][1] = acc[r][p][2] = acc[r][p][3] = 0.f;
    int cmax = cnt[0];
#pragma unroll
    for (int r = 1; r < R; ++r) cmax = max(cmax, cnt[r]);
    for (int c0 = 0; c0 < cmax; c0 += 32) {
      int2 ed[R];
#pragma unroll
      for (int r = 0; r < R; ++r) ed[r] = c0 + lane < cnt[r] ? a.csc_dst[e0[r] + c0 + lane] : make_int2(0, 1);
      const int m = min(32, cmax - c0);
      for (int j = 0; j < m; ++j) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int v = __shfl_sync(0xffffffffu, ed[r].x, j);
          const float fdeg = float(__shfl_sync(0xffffffffu, ed[r].y, j));
          if (c0 + j >= cnt[r]) continue;
          const float rc = __frcp_rn(fdeg);
          const float* zr = a.dz + int64_t(v) * a.dz_pitch;
#pragma unroll
          for (int p = 0; p < VPL; ++p) {
            const int jv = lane + 32 * p;
            if (jv < V) {
              const float4 z = *reinterpret_cast<const float4*>(zr + jv * 4);
              if (a.dz_scaled) {
                acc[r][p][0] += z.x; acc[r][p][1] += z.y; acc[r][p][2] += z.z; acc[r][p][3] += z.w;
              } else {
                acc[r][p][0] += div_rn_rcp(z.x, fdeg, rc);
                acc[r][p][1] += div_rn_rcp(z.y, fdeg, rc);
                acc[r][p][2] += div_rn_rcp(z.z, fdeg, rc);
                acc[r][p][3] += div_rn_rcp(z.w, fdeg, rc);
              }
            }
          }
        }
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r;
      if (u >= rows_out) continue;
#pragma unroll
      for (int p = 0; p < VPL; ++p) {
        const int j = lane + 32 * p;
        if (j >= V) continue;
        const uint32_t kp = (u < n) ? decode_mask<MS>(mraw[r][p]) : 0u;
        const float4 g = make_float4(kp & 1u ? acc[r][p][0] : 0.f, kp & 2u ? acc[r][p][1] : 0.f,
                                     kp & 4u ? acc[r][p][2] : 0.f, kp & 8u ? acc[r][p][3] : 0.f);
        const int c0 = j * 4;
        if (a.g && u < n) *reinterpret_cast<float4*>(a.g + u * a.g_pitch + c0) = g;
        if (a.gb) {
          uint16_t* o = a.gb + u * a.gb_pitch + c0;
          if (c0 + 4 <= a.dim) {
            *reinterpret_cast<uint2*>(o) = make_uint2(pack_bf16x2(g.x, g.y), pack_bf16x2(g.z, g.w));
          } else {
            const float w[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
            for (int q = 0; q < 4; ++q)
              if (c0 + q < a.dim) {
                __nv_bfloat16 hh = __float2bfloat16_rn(w[q]);
                o[q] = *reinterpret_cast<uint16_t*>(&hh);
              }
          }
        }
      }
    }
  }
}

// bf16 dZ / deg rows (reading R13), bf16 G, ReLU mask from bf16 H: a lane owns 8
// columns (one 16-B load per in-edge), R source rows in flight per warp; the mask is
// applied to the packed bf16 pairs with one AND against a per-half compare of H's bits
// (bf16 > 0 <=> its 16-bit pattern is a positive signed integer).
template <int VP, int R>
__global__ void __launch_bounds__(256) pull_bwd_b8_kernel(PullArgs a) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n = *a.n_src;
  const int V8 = a.dim >> 3;                      // dim % 8 == 0 (checked at launch)
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  const int64_t rows_out = std::min<int64_t>(a.max_src, round_up(n, 64));
  for (int64_t u0 = ((int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5) * R; u0 < rows_out; u0 += nwarps * R) {
    int e0[R], cnt[R];
    uint4 hm[R][VP];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r;
      e0[r] = 0; cnt[r] = 0;
      if (u < n) { e0[r] = a.csc_ptr[u]; cnt[r] = a.csc_ptr[u + 1] - e0[r]; }
#pragma unroll
      for (int p = 0; p < VP; ++p) {
        const int j = lane + 32 * p;
        hm[r][p] = (u < n && j < V8) ? __ldg(reinterpret_cast<const uint4*>(a.hb + u * a.hb_pitch + j * 8))
                                     : make_uint4(0, 0, 0, 0);
      }
    }
    float acc[R][VP][8];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int p = 0; p < VP; ++p)
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[r][p][q] = 0.f;
    int cmax = cnt[0];
#pragma unroll
    for (int r = 1; r < R; ++r) cmax = max(cmax, cnt[r]);
    for (int c0 = 0; c0 < cmax; c0 += 32) {
      int v[R];
#pragma unroll
      for (int r = 0; r < R; ++r) v[r] = c0 + lane < cnt[r] ? a.csc_dst[e0[r] + c0 + lane].x : 0;
      const int m = min(32, cmax - c0);
      for (int e = 0; e < m; ++e) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int w = __shfl_sync(0xffffffffu, v[r], e);
          if (c0 + e >= cnt[r]) continue;
#pragma unroll
          for (int p = 0; p < VP; ++p) {
            const int j = lane + 32 * p;
            if (j < V8) {
              const uint4 z = *reinterpret_cast<const uint4*>(a.dzb + int64_t(w) * a.dzb_pitch + j * 8);
              accumulate_bf16x8(acc[r][p], z);
            }
          }
        }
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r;
      if (u >= rows_out) continue;
#pragma unroll
      for (int p = 0; p < VP; ++p) {
        const int j = lane + 32 * p;
        if (j >= V8) continue;
        const float* x = acc[r][p];
        const uint4 o = make_uint4(pack_bf16x2(x[0], x[1]) & __vcmpgts2(hm[r][p].x, 0u),
                                   pack_bf16x2(x[2], x[3]) & __vcmpgts2(hm[r][p].y, 0u),
                                   pack_bf16x2(x[4], x[5]) & __vcmpgts2(hm[r][p].z, 0u),
                                   pack_bf16x2(x[6], x[7]) & __vcmpgts2(hm[r][p].w, 0u));
        *reinterpret_cast<uint4*>(a.gb + u * a.gb_pitch + j * 8) = o;
      }
    }
  }
}

// The same pull as a resident wave of warps, each streaming row groups with the next
// group's CSC bounds and its first 32 in-edges loaded one iteration ahead: a row group's
// dependent chain (CSC pointer -> in-edge -> dZ row) shrinks to the dZ row loads, where the
// block-per-group form paid all three round trips per group (layer-1 rows have ~1.3
// in-edges each, so the chain, not the bytes, set the time).
template <int VP, int R, int EB, bool BITS, int MINB = 4>
__global__ void __launch_bounds__(256, MINB) pull_bwd_b8_pf_kernel(PullArgs a) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n = *a.n_src;
  const int V8 = a.dim >> 3;
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  const int64_t rows_out = std::min<int64_t>(a.max_src, round_up(n, 64));
  int64_t u0 = ((int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5) * R;
  // each lane's column base in the dZ rows as an opaque 64-bit value (lanes past the row's
  // vectors read vector 0: in bounds, never stored)
  const uint32_t zrb = uint32_t(a.dzb_pitch * 2);
  uint64_t zb[VP];
#pragma unroll
  for (int p = 0; p < VP; ++p) {
    const int j = lane + 32 * p;
    asm("mov.b64 %0, %1;" : "=l"(zb[p]) : "l"(reinterpret_cast<uint64_t>(a.dzb) + uint64_t(j < V8 ? j : 0) * 16u));
  }
  int e0[R], cnt[R], vv[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const int64_t u = u0 + r;
    e0[r] = 0; cnt[r] = 0;
    if (u < n) { e0[r] = a.csc_ptr[u]; cnt[r] = a.csc_ptr[u + 1] - e0[r]; }
  }
#pragma unroll
  for (int r = 0; r < R; ++r) vv[r] = lane < cnt[r] ? a.csc_dst[e0[r] + lane].x : 0;
  for (; u0 < rows_out; u0 += nwarps * R) {
    uint4 hm[R][VP];
    int e0n[R], cntn[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r, un = u0 + nwarps * R + r;
#pragma unroll
      for (int p = 0; p < VP; ++p) {
        const int j = lane + 32 * p;
        if constexpr (BITS) {
          // the lane's 8 ReLU bits (one byte of the row's mask words) as positive bf16 halves
          // for the same packed-pair compare below
          uint32_t b = 0;
          if (u < n && j < V8) b = uint32_t(__ldg(a.mask + u * a.mask_pitch + (j >> 1))) >> (8 * (j & 1));
          hm[r][p] = make_uint4((b & 1u) | ((b & 2u) << 15), ((b >> 2) & 1u) | (((b >> 3) & 1u) << 16),
                                ((b >> 4) & 1u) | (((b >> 5) & 1u) << 16), ((b >> 6) & 1u) | (((b >> 7) & 1u) << 16));
        } else {
          hm[r][p] = (u < n && j < V8) ? __ldg(reinterpret_cast<const uint4*>(a.hb + u * a.hb_pitch + j * 8))
                                       : make_uint4(0, 0, 0, 0);
        }
      }
      e0n[r] = 0; cntn[r] = 0;
      if (un < n) { e0n[r] = a.csc_ptr[un]; cntn[r] = a.csc_ptr[un + 1] - e0n[r]; }
    }
    float acc[R][VP][8];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int p = 0; p < VP; ++p)
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[r][p][q] = 0.f;
    int cmax = cnt[0];
#pragma unroll
    for (int r = 1; r < R; ++r) cmax = max(cmax, cnt[r]);
    for (int c0 = 0; c0 < cmax; c0 += 32) {
      int v[R];
#pragma unroll
      for (int r = 0; r < R; ++r)
        v[r] = c0 == 0 ? vv[r] : (c0 + lane < cnt[r] ? a.csc_dst[e0[r] + c0 + lane].x : 0);
      const int m = min(32, cmax - c0);
      // EB in-edges of every row of the group in flight at once (predicated loads; the
      // rows average ~1.3 in-edges, so one batch usually covers the group)
#pragma unroll 1
      for (int eb = 0; eb < m; eb += EB) {
        uint4 z[EB][R][VP];
        bool ok[EB][R];
#pragma unroll
        for (int q = 0; q < EB; ++q)
#pragma unroll
          for (int r = 0; r < R; ++r) {
            const int e = eb + q;
            const int w = __shfl_sync(0xffffffffu, v[r], e & 31);
            ok[q][r] = e < m && c0 + e < cnt[r];
            // the row is always a valid one (lanes past a row's count hold id 0), so the
            // load is unconditional: one IMAD.WIDE off the lane's column base, the value
            // zeroed by selects where the edge is padding, the adds unconditional
#pragma unroll
            for (int p = 0; p < VP; ++p) {
              const uint4 t = __ldg(reinterpret_cast<const uint4*>(zb[p] + uint64_t(uint32_t(w)) * zrb));
              z[q][r][p] = ok[q][r] ? t : make_uint4(0, 0, 0, 0);
            }
          }
#pragma unroll
        for (int q = 0; q < EB; ++q)
#pragma unroll
          for (int r = 0; r < R; ++r)
#pragma unroll
            for (int p = 0; p < VP; ++p) accumulate_bf16x8(acc[r][p], z[q][r][p]);
      }
    }
    // the next group's first in-edges (its CSC bounds arrived during this group's sums)
#pragma unroll
    for (int r = 0; r < R; ++r) {
      e0[r] = e0n[r]; cnt[r] = cntn[r];
      vv[r] = lane < cnt[r] ? a.csc_dst[e0[r] + lane].x : 0;
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t u = u0 + r;
      if (u >= rows_out) continue;
#pragma unroll
      for (int p = 0; p < VP; ++p) {
        const int j = lane + 32 * p;
        if (j >= V8) continue;
        const float* x = acc[r][p];
        const uint4 o = make_uint4(pack_bf16x2(x[0], x[1]) & __vcmpgts2(hm[r][p].x, 0u),
                                   pack_bf16x2(x[2], x[3]) & __vcmpgts2(hm[r][p].y, 0u),
                                   pack_bf16x2(x[4], x[5]) & __vcmpgts2(hm[r][p].z, 0u),
                                   pack_bf16x2(x[6], x[7]) & __vcmpgts2(hm[r][p].w, 0u));
        *reinterpret_cast<uint4*>(a.gb + u * a.gb_pitch + j * 8) = o;
      }
    }
  }
}

cudaError_t launch_pull_bwd(const PullArgs& a, cudaStream_t st) {
  if (a.dim > 512) {   // wide rows: column chunks of 512 (128 fp32 vectors per lane group)
    for (int c0 = 0; c0 < a.dim; c0 += 512) {
      PullArgs b = a;
      b.dim = std::min(512, a.dim - c0);
      b.dz = a.dz + c0;
      if (a.h) b.h = a.h + c0;
      if (a.hb) b.hb = a.hb + c0;
      if (a.dzb) b.dzb = a.dzb + c0;
      if (a.mask) b.mask = a.mask + c0 / 16;
      if (a.g) b.g = a.g + c0;
      if (a.gb) b.gb = a.gb + c0;
      cudaError_t e = launch_pull_bwd(b, st);
      if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
  }
  const int V = int(ceil_div(a.dim, 4));
  if ((a.dz_pitch & 3) || (a.h_pitch & 3) || (a.g && (a.g_pitch & 3)) || (a.gb && (a.gb_pitch & 3)))
    return cudaErrorInvalidValue;
  constexpr int R = 2;   // rows in flight per warp
  if (a.dzb) {            // reading R13 (bf16 mode): bf16 dZ, bf16 G, mask from bf16 H
    if (!a.gb || a.g || !a.hb || (a.dim & 7) || (a.dzb_pitch & 7) || (a.hb_pitch & 7) || (a.gb_pitch & 7))
      return cudaErrorInvalidValue;
    static const int rr = [] { const char* e = std::getenv("APT_PULL_ROWS"); return e ? atoi(e) : 2; }();
    const int Rr = rr == 4 ? 4 : 2;
    // APT_PULL_BPSM: grid cap in blocks per SM (A/B knob)
    static const int bpsm = [] { const char* e = std::getenv("APT_PULL_BPSM"); return e ? atoi(e) : 16; }();
    const int64_t blocks = std::max<int64_t>(
        1, std::min<int64_t>(ceil_div(ceil_div(round_up(a.max_src, 64), Rr) * 32, 256), int64_t(num_sms()) * bpsm));
    const int V8 = a.dim >> 3;
    static const int pf = [] { const char* e = std::getenv("APT_PULL_PF"); return e ? atoi(e) : 1; }();
    if (pf && V8 <= 32) {
      // one resident wave (APT_PULL_PF_BPSM caps blocks per SM: A/B knob)
      static const int pbpsm = [] { const char* e = std::getenv("APT_PULL_PF_BPSM"); return e ? atoi(e) : 0; }();
      // in-edges in flight per row (APT_PULL_EB) x rows per warp (APT_PULL_ROWS): A/B knobs
      static const int eb = [] { const char* e = std::getenv("APT_PULL_EB"); return e ? atoi(e) : 1; }();   // 1 / 2 / 4: 0.1627 / 0.1673 / 0.1786 ms (A/B)
      // APT_PULL_MINB: blocks per SM the register allocation must allow (A/B)
      static const int pminb = [] { const char* e = std::getenv("APT_PULL_MINB"); return e ? atoi(e) : 0; }();
      auto kern = (!a.mask && Rr == 2 && rr != 1 && eb <= 1 && pminb >= 5)
                  ? (pminb >= 6 ? pull_bwd_b8_pf_kernel<1, 2, 1, false, 6> : pull_bwd_b8_pf_kernel<1, 2, 1, false, 5>)
                : a.mask ? pull_bwd_b8_pf_kernel<1, 2, 1, true>
                : Rr == 4 ? pull_bwd_b8_pf_kernel<1, 4, 1, false>
                : (rr == 1 ? (eb >= 4 ? pull_bwd_b8_pf_kernel<1, 1, 4, false> : pull_bwd_b8_pf_kernel<1, 1, 2, false>)
                : (eb >= 4 ? pull_bwd_b8_pf_kernel<1, 2, 4, false> : eb == 2 ? pull_bwd_b8_pf_kernel<1, 2, 2, false>
                : pull_bwd_b8_pf_kernel<1, 2, 1, false>));
      const int Rk = rr == 1 ? 1 : Rr;
      const int64_t pblocks = grid_cap(ceil_div(ceil_div(round_up(a.max_src, 64), Rk) * 32, 256),
                                       pbpsm > 0 ? pbpsm : resident_blocks(kern, 256));
      launch_pdl(kern, dim3(pblocks), dim3(256), 0, st, a);
      return cudaGetLastError();
    }
    if (Rr == 4) {
      if (V8 <= 32) launch_pdl(pull_bwd_b8_kernel<1, 4>, dim3(blocks), dim3(256), 0, st, a);
      else launch_pdl(pull_bwd_b8_kernel<2, 4>, dim3(blocks), dim3(256), 0, st, a);
    } else {
      if (V8 <= 32) launch_pdl(pull_bwd_b8_kernel<1, 2>, dim3(blocks), dim3(256), 0, st, a);
      else launch_pdl(pull_bwd_b8_kernel<2, 2>, dim3(blocks), dim3(256), 0, st, a);
    }
    return cudaGetLastError();
  }
  const int64_t blocks =
      std::max<int64_t>(1, std::min<int64_t>(ceil_div(ceil_div(round_up(a.max_src, 64), R) * 32, 256), int64_t(num_sms()) * 16));
  const int ms = a.mask ? 1 : a.hb ? 3 : a.h ? 2 : 0;
  auto go = [&](auto vpl) {
    constexpr int VP = decltype(vpl)::value;
    if (ms == 0) launch_pdl(pull_bwd_kernel<VP, R, 0>, dim3(blocks), dim3(256), 0, st, a);
    else if (ms == 1) launch_pdl(pull_bwd_kernel<VP, R, 1>, dim3(blocks), dim3(256), 0, st, a);
    else if (ms == 2) launch_pdl(pull_bwd_kernel<VP, R, 2>, dim3(blocks), dim3(256), 0, st, a);
    else launch_pdl(pull_bwd_kernel<VP, R, 3>, dim3(blocks), dim3(256), 0, st, a);
  };
  if (V <= 32) go(std::integral_constant<int, 1>{});
  else if (V <= 64) go(std::integral_constant<int, 2>{});
  else if (V <= 128) go(std::integral_constant<int, 4>{});
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

}  // namespace apt
