// outlayer.cu -- the output layer K of the step in one kernel (S10, bf16 mode):
//
//   Z_K  = mean over the sampled in-edges of H_{K-1} (bf16 rows)        (Eq. 1)
//   pre  = Z_K W_K^T + b_K (logits, no activation: reading Z9)
//   loss += sum_s CE(pre_s, y_s) / |global batch|                      (reading Z20)
//   G_K  = dL/dpre (fp32 + its bf16 copy for the tcgen05 weight gradient)
//   dZ_K = (G_K W_K) / deg                                              (backward of the
//          projection, pre-divided by the row's sampled degree for the pull-form mean
//          backward, as the tcgen05 epilogue does for the other layers)
//
// Why one kernel: the output layer is tiny (B rows x <= 64 classes) and its five
// kernels (mean, projection, CE, dZ projection, ...) were each a chain of dependent
// loads with a launch/drain around it -- latency, not bandwidth.  Here a CTA owns 8
// seed rows end to end: each warp gathers one row's neighbours (16-B bf16 vectors,
// 4 edges in flight per lane), the CTA holds W_K (fp32, padded rows: conflict-free)
// and the 8 rows of Z in shared memory, a lane computes two classes' logits, the
// warp does the row's softmax / CE, then the lane computes 8 columns of dZ.  The
// arithmetic matches the unfused path: fp32 sums and the IEEE division of the mean
// (reading O5), bf16 Z and W with fp32 accumulation, dZ from the bf16-rounded G.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>

namespace apt {

namespace {
constexpr int OL_ROWS = 8;        // seed rows per CTA (one warp each)
constexpr int OL_MAX_OUT = 64;    // classes
constexpr int OL_MAX_IN = 256;    // input width (32 lanes x 8 bf16)
constexpr int OL_WP = OL_MAX_IN + 1;   // fp32 smem pitch of W rows (bank-conflict free)
}  // namespace

__global__ void __launch_bounds__(256) outlayer_kernel(OutLayerArgs a) {
  extern __shared__ float ol_smem[];
  float* Ws = ol_smem;                                   // [d_out][OL_WP]
  float* Zs = Ws + OL_MAX_OUT * OL_WP;                   // [OL_ROWS][OL_MAX_IN]
  float* Gs = Zs + OL_ROWS * OL_MAX_IN;                  // [OL_ROWS][OL_MAX_OUT] bf16-rounded g
  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int din = a.d_in, dout = a.d_out;
  // W_K does not change within the step (SGD runs at its end): stage it before the PDL wait
  // 16-B vectors of the bf16 rows (wb_pitch is a multiple of 8; the padding columns
  // are zero), all of a thread's loads in flight at once
  {
    const int vpr = int(a.wb_pitch / 8), nv = dout * vpr;
    constexpr int PER = (OL_MAX_OUT * OL_MAX_IN / 8 + 255) / 256;
    uint4 w[PER];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const int i = threadIdx.x + 256 * j;
      w[j] = i < nv ? ld_nc_v4(a.Wb + int64_t(i / vpr) * a.wb_pitch + (i % vpr) * 8) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const int i = threadIdx.x + 256 * j;
      if (i >= nv) continue;
      float* o = Ws + (i / vpr) * OL_WP + (i % vpr) * 8;
      o[0] = bf16_lo(w[j].x); o[1] = bf16_hi(w[j].x); o[2] = bf16_lo(w[j].y); o[3] = bf16_hi(w[j].y);
      o[4] = bf16_lo(w[j].z); o[5] = bf16_hi(w[j].z); o[6] = bf16_lo(w[j].w); o[7] = bf16_hi(w[j].w);
    }
  }
  pdl_wait();
  pdl_launch();
  __syncthreads();
  const int64_t n = *a.n_dst;
  const int64_t r = int64_t(blockIdx.x) * OL_ROWS + warp;
  const int64_t tail = std::min<int64_t>(a.max_dst, round_up(n, 64));
  if (r >= n) {   // zero Gb over the last 64-row block (the tcgen05 weight gradient reads whole blocks)
    if (r < tail)
      for (int c = lane; c < a.gb_pitch; c += 32) a.Gb[r * a.gb_pitch + c] = 0;
    return;       // no __syncthreads below involves this warp's row
  }
  // ---- mean of the row's sampled in-neighbours (H_{K-1} bf16 rows, 16-B vectors)
  const int V = (din + 7) / 8;
  const int e0 = a.indptr[r], cnt = a.indptr[r + 1] - e0;
  float acc[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) acc[q] = 0.f;
  for (int c0 = 0; c0 < cnt; c0 += 32) {
    const int u_l = c0 + lane < cnt ? a.indices[e0 + c0 + lane] : 0;
    const int m = min(32, cnt - c0);
    for (int j = 0; j < m; j += 4) {
      uint4 v[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int u = __shfl_sync(0xffffffffu, u_l, (j + q) & 31);
        v[q] = (j + q < m && lane < V) ? ld_nc_v4(a.xb + int64_t(u) * a.x_pitch + lane * 8) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        acc[0] += bf16_lo(v[q].x); acc[1] += bf16_hi(v[q].x);
        acc[2] += bf16_lo(v[q].y); acc[3] += bf16_hi(v[q].y);
        acc[4] += bf16_lo(v[q].z); acc[5] += bf16_hi(v[q].z);
        acc[6] += bf16_lo(v[q].w); acc[7] += bf16_hi(v[q].w);
      }
    }
  }
  const float fdeg = float(cnt);
  const float rdeg = cnt > 0 ? __frcp_rn(fdeg) : 0.f;
  float* zrow = Zs + warp * OL_MAX_IN;
  if (lane < V) {
    float z[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const float zz = cnt > 0 ? div_rn_rcp(acc[q], fdeg, rdeg) : 0.f;
      z[q] = bf16_bits_to_float(bf16_bits(zz));     // Z is stored (and projected) in bf16
    }
    uint16_t* zo = a.Zb + r * a.zb_pitch + lane * 8;
    if (lane * 8 + 8 <= din) {
      *reinterpret_cast<uint4*>(zo) = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]),
                                                 pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
    } else {
      for (int q = 0; q < 8 && lane * 8 + q < din; ++q) zo[q] = bf16_bits(z[q]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q)
      if (lane * 8 + q < din) zrow[lane * 8 + q] = z[q];
  }
  if (lane == 0) a.Zb[r * a.zb_pitch + din] = 0x3F80;   // bf16 1.0: the bias-gradient column
  __syncwarp();
  // ---- logits: lane owns classes lane and lane + 32
  float lg[2];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int c = lane + 32 * h;
    float s = 0.f;
    if (c < dout) {   // four independent partial sums (FMA latency), summed in a fixed order
      const float* w = Ws + c * OL_WP;
      float p0 = 0.f, p1 = 0.f, p2 = 0.f, p3 = 0.f;
      int k = 0;
      for (; k + 4 <= din; k += 4) {
        p0 = fmaf(zrow[k], w[k], p0); p1 = fmaf(zrow[k + 1], w[k + 1], p1);
        p2 = fmaf(zrow[k + 2], w[k + 2], p2); p3 = fmaf(zrow[k + 3], w[k + 3], p3);
      }
      for (; k < din; ++k) p0 = fmaf(zrow[k], w[k], p0);
      s = ((p0 + p1) + (p2 + p3)) + a.bias[c];
    }
    lg[h] = s;
  }
  // ---- softmax cross entropy of the row (loss summed over seeds / |global batch|)
  float mx = -INFINITY;
#pragma unroll
  for (int h = 0; h < 2; ++h)
    if (lane + 32 * h < dout) mx = fmaxf(mx, lg[h]);
  mx = warp_max(mx);
  float se = 0.f;
#pragma unroll
  for (int h = 0; h < 2; ++h)
    if (lane + 32 * h < dout) se += expf(lg[h] - mx);
  se = warp_sum(se);
  const float lse = mx + logf(se);
  const int y = a.labels[a.seeds[r]];
  const float inv_n = 1.0f / float(max(1, *a.n_global));
  float* grow = Gs + warp * OL_MAX_OUT;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int c = lane + 32 * h;
    if (c >= dout) continue;
    if (c == y) atomicAdd(a.loss, (lse - lg[h]) * inv_n);
    const float g = (expf(lg[h] - lse) - (c == y ? 1.f : 0.f)) * inv_n;
    a.H[r * a.h_pitch + c] = lg[h];
    a.G[r * a.g_pitch + c] = g;
    const uint16_t gb = bf16_bits(g);
    a.Gb[r * a.gb_pitch + c] = gb;
    grow[c] = bf16_bits_to_float(gb);                 // dZ uses the bf16 G (reading R4)
  }
  for (int c = dout + lane; c < a.gb_pitch; c += 32) a.Gb[r * a.gb_pitch + c] = 0;
  __syncwarp();
  // ---- dZ = (G W) / deg: lane owns columns lane + 32 j
  float* dz = a.dZ + r * a.dz_pitch;
  float s[OL_MAX_IN / 32];
#pragma unroll
  for (int j = 0; j < OL_MAX_IN / 32; ++j) s[j] = 0.f;
  for (int c = 0; c < dout; ++c) {   // eight independent chains (one per owned column)
    const float gc = grow[c];
    const float* w = Ws + c * OL_WP + lane;
#pragma unroll
    for (int j = 0; j < OL_MAX_IN / 32; ++j) s[j] = fmaf(gc, w[32 * j], s[j]);
  }
#pragma unroll
  for (int j = 0; j < OL_MAX_IN / 32; ++j) {
    const int k = lane + 32 * j;
    if (k < din) dz[k] = cnt > 0 ? div_rn_rcp(s[j], fdeg, rdeg) : 0.f;
  }
}

int outlayer_supported(int d_in, int d_out) { return d_in >= 1 && d_in <= OL_MAX_IN && d_out >= 1 && d_out <= OL_MAX_OUT; }

cudaError_t launch_outlayer(const OutLayerArgs& a, cudaStream_t st) {
  if (!outlayer_supported(a.d_in, a.d_out) || (a.x_pitch % 8) || a.gb_pitch < a.d_out) return cudaErrorInvalidValue;
  const size_t smem = sizeof(float) * (OL_MAX_OUT * OL_WP + OL_ROWS * OL_MAX_IN + OL_ROWS * OL_MAX_OUT);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(outlayer_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    attr = true;
  }
  const int64_t blocks = std::max<int64_t>(1, ceil_div(a.max_dst, OL_ROWS));
  launch_pdl(outlayer_kernel, dim3(blocks), dim3(256), smem, st, a);
  return cudaGetLastError();
}

}  // namespace apt
