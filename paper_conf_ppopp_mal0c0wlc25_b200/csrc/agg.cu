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

namespace apt {

template <int EPV>
__device__ __forceinline__ void accumulate_vec(float* acc, uint4 raw) {
  if constexpr (EPV == 8) {
    acc[0] += bf16_lo(raw.x); acc[1] += bf16_hi(raw.x);
    acc[2] += bf16_lo(raw.y); acc[3] += bf16_hi(raw.y);
    acc[4] += bf16_lo(raw.z); acc[5] += bf16_hi(raw.z);
    acc[6] += bf16_lo(raw.w); acc[7] += bf16_hi(raw.w);
  } else {
    acc[0] += __uint_as_float(raw.x); acc[1] += __uint_as_float(raw.y);
    acc[2] += __uint_as_float(raw.z); acc[3] += __uint_as_float(raw.w);
  }
}

struct EllFstoreSrc {
  const int32_t* cnt; const int32_t* nbr; int k;
  FeatView fv;
  __device__ int64_t begin(int64_t i) const { return i * k; }
  __device__ int64_t end(int64_t i) const { return i * k + cnt[i]; }
  __device__ int node(int64_t e) const { return nbr[e]; }
  __device__ const char* row(int u) const {
    if (fv.part) {
      const int o = fv.part[u];
      return reinterpret_cast<const char*>(fv.base[o]) + int64_t(fv.lrow[u]) * fv.pitch * (fv.dtype == kBF16 ? 2 : 4);
    }
    return reinterpret_cast<const char*>(fv.base[0]) + int64_t(u) * fv.pitch * (fv.dtype == kBF16 ? 2 : 4);
  }
};

struct CsrSrc {
  const int32_t* indptr; const int32_t* indices; const float* x; int64_t pitch;
  __device__ int64_t begin(int64_t i) const { return indptr[i]; }
  __device__ int64_t end(int64_t i) const { return indptr[i + 1]; }
  __device__ int node(int64_t e) const { return indices[e]; }
  __device__ const char* row(int u) const { return reinterpret_cast<const char*>(x + int64_t(u) * pitch); }
};

// EPV: elements per 16-B vector (8 = bf16 input, 4 = fp32 input); VPL: vectors per lane.
template <int EPV, int VPL, class Src>
__global__ void __launch_bounds__(256) agg_kernel(AggArgs a, Src src) {
  const int lane = lane_id();
  const int64_t n_dst = *a.n_dst;
  const int V = int(ceil_div(a.dim, EPV));
  const int G = (VPL == 1 && V <= 16) ? (32 / V) : 1;      // lane groups (edges in flight)
  const int g = (VPL == 1) ? lane / V : 0;
  const int jv = (VPL == 1) ? lane - g * V : lane;          // first vector of this lane
  const bool active = (VPL == 1) ? (g < G) : true;
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n_dst; i += nwarps) {
    float acc[VPL][EPV];
#pragma unroll
    for (int p = 0; p < VPL; ++p)
#pragma unroll
      for (int q = 0; q < EPV; ++q) acc[p][q] = 0.f;
    const int64_t e0 = src.begin(i), e1 = src.end(i);
    int deg = int(e1 - e0);
    if (a.deg_override) deg = a.deg_override[i];
    if (active) {
      int64_t e = e0 + g;
      // two edges per group per iteration: 2*G*V independent 16-B loads per warp
      for (; e + G < e1; e += 2 * G) {
        const int u0 = src.node(e), u1 = src.node(e + G);
        const bool k0 = !a.filt_part || a.filt_part[u0] == a.keep_part;
        const bool k1 = !a.filt_part || a.filt_part[u1] == a.keep_part;
        const char* r0 = src.row(u0);
        const char* r1 = src.row(u1);
        uint4 v0[VPL], v1[VPL];
#pragma unroll
        for (int p = 0; p < VPL; ++p) {
          const int j = jv + p * 32;
          v0[p] = (k0 && j < V) ? ld_nc_v4(r0 + int64_t(j) * 16) : make_uint4(0, 0, 0, 0);
          v1[p] = (k1 && j < V) ? ld_nc_v4(r1 + int64_t(j) * 16) : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int p = 0; p < VPL; ++p) { accumulate_vec<EPV>(acc[p], v0[p]); accumulate_vec<EPV>(acc[p], v1[p]); }
      }
      if (e < e1) {
        const int u0 = src.node(e);
        if (!a.filt_part || a.filt_part[u0] == a.keep_part) {
          const char* r0 = src.row(u0);
#pragma unroll
          for (int p = 0; p < VPL; ++p) {
            const int j = jv + p * 32;
            if (j < V) accumulate_vec<EPV>(acc[p], ld_nc_v4(r0 + int64_t(j) * 16));
          }
        }
      }
    }
    if (VPL == 1) {   // fold the G lane groups into group 0 (fixed order: deterministic)
      for (int s = 1; s < G; ++s) {
#pragma unroll
        for (int q = 0; q < EPV; ++q) {
          const float o = __shfl_sync(0xffffffffu, acc[0][q], (lane + s * V) & 31);
          if (g == 0 && lane + s * V < 32) acc[0][q] += o;
        }
      }
    }
    if (g != 0 || !active) continue;
    if (a.z_ones && lane == 0) a.z_bf16[i * a.z_bf16_pitch + a.dim] = 0x3F80;   // bf16 1.0: bias-gradient column
    const float fdeg = float(deg);
#pragma unroll
    for (int p = 0; p < VPL; ++p) {
      const int j = jv + p * 32;
      if (j >= V) continue;
      float z[EPV];
#pragma unroll
      for (int q = 0; q < EPV; ++q) z[q] = deg > 0 ? __fdiv_rn(acc[p][q], fdeg) : 0.f;
      const int c0 = j * EPV;
      const bool full = c0 + EPV <= a.dim;
      if (a.z_f32) {
        float* o = a.z_f32 + i * a.z_f32_pitch + c0;
        if (full) {
#pragma unroll
          for (int q = 0; q < EPV; q += 4) *reinterpret_cast<float4*>(o + q) = make_float4(z[q], z[q + 1], z[q + 2], z[q + 3]);
        } else {
          for (int q = 0; q < EPV && c0 + q < a.dim; ++q) o[q] = z[q];
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
          for (int q = 0; q < EPV && c0 + q < a.dim; ++q) {
            __nv_bfloat16 h = __float2bfloat16_rn(z[q]);
            o[q] = *reinterpret_cast<uint16_t*>(&h);
          }
        }
      }
    }
  }
}

template <int EPV, class Src>
static cudaError_t dispatch_agg(const AggArgs& a, const Src& s, cudaStream_t st) {
  const int V = int(ceil_div(a.dim, EPV));
  const int threads = 256;
  int64_t blocks = ceil_div(a.max_dst * 32, threads);
  blocks = std::max<int64_t>(1, std::min<int64_t>(blocks, 148 * 16));
  if (V <= 32) agg_kernel<EPV, 1, Src><<<blocks, threads, 0, st>>>(a, s);
  else if (V <= 64) agg_kernel<EPV, 2, Src><<<blocks, threads, 0, st>>>(a, s);
  else if (V <= 128) agg_kernel<EPV, 4, Src><<<blocks, threads, 0, st>>>(a, s);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

cudaError_t launch_agg_fstore(const AggArgs& a, const FeatView& fv, cudaStream_t st) {
  EllFstoreSrc s{a.cnt, a.nbr, a.k, fv};
  AggArgs b = a;
  b.dim = fv.dim;
  return fv.dtype == kBF16 ? dispatch_agg<8>(b, s, st) : dispatch_agg<4>(b, s, st);
}

cudaError_t launch_agg_csr(const AggArgs& a, cudaStream_t st) {
  CsrSrc s{a.indptr, a.indices, a.x, a.x_pitch};
  return dispatch_agg<4>(a, s, st);
}

// ---------------------------------------------------------------- backward
// dX[src_e] += dZ[v] / deg_s(v): one warp per dst, the dZ row held in registers,
// one 16-B vector red per lane per edge.
__global__ void __launch_bounds__(256) agg_bwd_kernel(const int32_t* __restrict__ indptr,
                                                      const int32_t* __restrict__ indices,
                                                      const int32_t* __restrict__ n_dst_p, const float* __restrict__ dz,
                                                      int64_t dz_pitch, int dim, float* __restrict__ dx,
                                                      int64_t dx_pitch) {
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
      const float a = __fdiv_rn(g.x, fdeg), b = __fdiv_rn(g.y, fdeg), c = __fdiv_rn(g.z, fdeg), d = __fdiv_rn(g.w, fdeg);
      for (int e = e0; e < e1; ++e) red_add_v4(dx + int64_t(indices[e]) * dx_pitch + j * 4, a, b, c, d);
    }
  }
}

cudaError_t launch_agg_bwd(const int32_t* indptr, const int32_t* indices, const int32_t* n_dst, int64_t max_dst,
                           const float* dz, int64_t dz_pitch, int dim, float* dx, int64_t dx_pitch, cudaStream_t st) {
  int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(max_dst * 32, 256), 148 * 16));
  agg_bwd_kernel<<<blocks, 256, 0, st>>>(indptr, indices, n_dst, dz, dz_pitch, dim, dx, dx_pitch);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- gather
__global__ void gather_kernel(FeatView fv, const int32_t* __restrict__ ids, const int32_t* __restrict__ n_p,
                              int64_t n_static, char* __restrict__ out, int64_t out_pitch_bytes) {
  const int64_t n = n_p ? int64_t(*n_p) : n_static;
  const int esz = fv.dtype == kBF16 ? 2 : 4;
  const int V = int(ceil_div(int64_t(fv.dim) * esz, 16));
  const int lane = lane_id();
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n; i += nwarps) {
    const int u = ids[i];
    const char* row = fv.part ? reinterpret_cast<const char*>(fv.base[fv.part[u]]) + int64_t(fv.lrow[u]) * fv.pitch * esz
                              : reinterpret_cast<const char*>(fv.base[0]) + int64_t(u) * fv.pitch * esz;
    for (int j = lane; j < V; j += 32)
      *reinterpret_cast<uint4*>(out + i * out_pitch_bytes + j * 16) = ld_nc_v4(row + j * 16);
  }
}

cudaError_t launch_gather(const FeatView& fv, const int32_t* ids, const int32_t* n_dev, int64_t max_n, void* out,
                          int64_t out_pitch, cudaStream_t st) {
  int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(max_n * 32, 256), 148 * 16));
  const int esz = fv.dtype == kBF16 ? 2 : 4;
  gather_kernel<<<blocks, 256, 0, st>>>(fv, ids, n_dev, max_n, reinterpret_cast<char*>(out), out_pitch * esz);
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
  int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(n * pitch, 256), 148 * 64));
  fill_features_kernel<<<blocks, 256, 0, st>>>(shard, dt == kBF16, pitch, col0, ncols, ids, n,
                                               philox_key(seed, kDomFeat));
  return cudaGetLastError();
}

}  // namespace apt
