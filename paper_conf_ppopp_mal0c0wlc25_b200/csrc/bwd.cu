// bwd.cu -- the mean's backward as a gather (S10): G_{l-1} = relu'(H_{l-1}) * D^T (dZ_l / deg).
//
// The scatter form (dX[src_e] += dZ[v]/deg(v), agg_bwd_kernel) needs a zeroed fp32
// buffer, ~E red.v4 atomics and a separate masking/bf16 pass.  Here the sampled
// block is transposed once per step (counting sort: count, scan, fill -- built on
// the side stream while the forward runs) and every source row pulls its in-edges:
// one pass reads dZ (L2-resident), the ReLU mask from H, and writes G (fp32) and/or
// its bf16 copy directly; no atomics, no zeroing.  Within a row the in-edges are
// summed in a fixed (CSC) order.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>

namespace apt {

cudaError_t launch_scan_counts(const int32_t* cnt, const int32_t* n_dev, int64_t max_n, int32_t* out, int32_t* total,
                               int32_t* ws, cudaStream_t st);

// in-degree of every local source of the block
__global__ void csc_count_kernel(const int32_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                 const int32_t* __restrict__ n_edges_p, int32_t* __restrict__ cnt) {
  APT_PDL_PROLOGUE();
  const int64_t E = *n_edges_p;
  for (int64_t e = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < E; e += int64_t(gridDim.x) * blockDim.x)
    atomicAdd(cnt + indices[e], 1);
}

// csc_dst[csc_ptr[u] + j] = v for the j-th in-edge (v, u); counts return to 0 (ready for the next step)
__global__ void csc_fill_kernel(const int32_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                const int32_t* __restrict__ n_dst_p, const int32_t* __restrict__ csc_ptr,
                                int32_t* __restrict__ cnt, int32_t* __restrict__ csc_dst) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_dst_p;
  for (int64_t v = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; v < n; v += int64_t(gridDim.x) * blockDim.x) {
    for (int e = indptr[v]; e < indptr[v + 1]; ++e) {
      const int u = indices[e];
      csc_dst[csc_ptr[u] + atomicSub(cnt + u, 1) - 1] = int32_t(v);
    }
  }
}

cudaError_t launch_csc_build(const CscArgs& a, cudaStream_t st) {
  const int64_t T = 256;
  const int64_t cap = a.grid_cap > 0 ? a.grid_cap : 148 * 16;
  const int64_t ge = std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.max_edges, T), cap));
  launch_pdl(csc_count_kernel, dim3(ge), dim3(T), 0, st, a.indptr, a.indices, a.n_edges, a.cnt);
  cudaError_t e = launch_scan_counts(a.cnt, a.n_src, a.max_src, a.csc_ptr, a.csc_total, a.ws, st);
  if (e != cudaSuccess) return e;
  const int64_t gd = std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.max_dst, T), cap));
  launch_pdl(csc_fill_kernel, dim3(gd), dim3(T), 0, st, a.indptr, a.indices, a.n_dst, a.csc_ptr, a.cnt, a.csc_dst);
  return cudaGetLastError();
}

// One warp per source row u (VPL float4 vectors per lane): g = sum over in-edges of
// dZ[v] / deg(v) (correctly rounded per term, reading O5), masked by H[u] > 0.
template <int VPL>
__global__ void __launch_bounds__(256) pull_bwd_kernel(PullArgs a) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n = *a.n_src;
  const int V = int(ceil_div(a.dim, 4));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  const int64_t rows_out = a.gb ? std::min<int64_t>(a.max_src, round_up(n, 64)) : n;
  for (int64_t u = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; u < rows_out; u += nwarps) {
    float acc[VPL][4];
#pragma unroll
    for (int p = 0; p < VPL; ++p) acc[p][0] = acc[p][1] = acc[p][2] = acc[p][3] = 0.f;
    if (u < n) {
      const int e0 = a.csc_ptr[u], e1 = a.csc_ptr[u + 1];
      for (int e = e0; e < e1; ++e) {
        const int v = a.csc_dst[e];
        const float fdeg = float(a.indptr[v + 1] - a.indptr[v]);
        const float r = __frcp_rn(fdeg);
        const float* zr = a.dz + int64_t(v) * a.dz_pitch;
#pragma unroll
        for (int p = 0; p < VPL; ++p) {
          const int j = lane + 32 * p;
          if (j < V) {
            const float4 z = *reinterpret_cast<const float4*>(zr + j * 4);
            acc[p][0] += div_rn_rcp(z.x, fdeg, r);
            acc[p][1] += div_rn_rcp(z.y, fdeg, r);
            acc[p][2] += div_rn_rcp(z.z, fdeg, r);
            acc[p][3] += div_rn_rcp(z.w, fdeg, r);
          }
        }
      }
    }
#pragma unroll
    for (int p = 0; p < VPL; ++p) {
      const int j = lane + 32 * p;
      if (j >= V) continue;
      float4 g = make_float4(acc[p][0], acc[p][1], acc[p][2], acc[p][3]);
      if (u < n && a.mask) {
        const uint32_t mw = uint32_t(a.mask[u * a.mask_pitch + (j * 4) / 16]) >> ((j * 4) & 15);
        if (!(mw & 1u)) g.x = 0.f;
        if (!(mw & 2u)) g.y = 0.f;
        if (!(mw & 4u)) g.z = 0.f;
        if (!(mw & 8u)) g.w = 0.f;
      } else if (u < n && a.h) {
        const float4 h = *reinterpret_cast<const float4*>(a.h + u * a.h_pitch + j * 4);
        if (!(h.x > 0.f)) g.x = 0.f;
        if (!(h.y > 0.f)) g.y = 0.f;
        if (!(h.z > 0.f)) g.z = 0.f;
        if (!(h.w > 0.f)) g.w = 0.f;
      }
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

cudaError_t launch_pull_bwd(const PullArgs& a, cudaStream_t st) {
  if (a.dim > 512) {   // wide rows: column chunks of 512 (128 fp32 vectors per lane group)
    for (int c0 = 0; c0 < a.dim; c0 += 512) {
      PullArgs b = a;
      b.dim = std::min(512, a.dim - c0);
      b.dz = a.dz + c0;
      if (a.h) b.h = a.h + c0;
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
  const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(round_up(a.max_src, 64) * 32, 256), 148 * 16));
  if (V <= 32) launch_pdl(pull_bwd_kernel<1>, dim3(blocks), dim3(256), 0, st, a);
  else if (V <= 64) launch_pdl(pull_bwd_kernel<2>, dim3(blocks), dim3(256), 0, st, a);
  else if (V <= 128) launch_pdl(pull_bwd_kernel<4>, dim3(blocks), dim3(256), 0, st, a);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

}  // namespace apt
