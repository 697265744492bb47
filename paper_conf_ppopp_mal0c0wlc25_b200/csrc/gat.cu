// gat.cu -- the GAT first layer under GDP / NFP / SNP / DNP.
//
// GAT [45] as the paper trains it (attention aggregation, hidden 8 x 4 heads)
// with readings G1-G4 (oracle/gat.py):
//   e_vu^h = LeakyReLU_0.2(a_src^h . W^h x_u + a_dst^h . W^h x_v),
//   alpha_vu^h = softmax_u(e_vu^h),  pre_v^h = W^h sum_u alpha_vu^h x_u  (+ b, ReLU).
//
// B200 design: the layer is evaluated "aggregate first" -- the score terms are dot
// products of the RAW feature row with w~^h = W^hT a^h (an H x d vector pair made
// once per step), so one fused gather kernel reads every sampled source row once
// and produces both the attention and the per-head weighted sums Z_v^h =
// sum_u alpha_vu^h x_u (online softmax: running max / sum per head, no second pass
// over the rows); the projection pre^h = W^h Z^h then runs per head on the items'
// Z.  This is the same structure as the SAGE layer (gather+mean, then projection),
// so every strategy of strategies.cu carries over (Fig. 5):
//   GDP  items = the rank's own rows, no exchange.
//   DNP  the owner of v has all of v's sources: full attention, h rows stored
//        straight into the requester's buffer ("friendly to attention").
//   SNP  owner c sees only its sources of v ("needs to pay extra
//        communication"): it keeps its partial softmax state (max m_c, sum S_c) and
//        its normalised partial Z_c, projects it, and ships (Q_c, m_c, S_c) to the
//        requester, which merges them with the online-softmax rule
//        out = sum_c S_c e^{m_c - m} Q_c / sum_c S_c e^{m_c - m} (one pass).
//        The dst term needs x_v: the owner reads it (local or NVLink peer row).
//   NFP  the scores are sums over the feature-column slices (P:225
//        SegmentedSDDMM): every owner adds its partial score of every edge into the
//        requester's score buffer (reduce), reads the full score back after a
//        barrier (broadcast) -- an all-reduce of the partial dot products -- then
//        aggregates its column slice and projects with its column slice of W.
// Backward, per owner item: gamma^h = W^hT g^h, dalpha = gamma^h . x_u (NFP:
// summed over slices like the scores), de = alpha (dalpha - t) with t = g . (pre -
// b) from the requester, ds = de * LeakyReLU'(e); dL/dw~_src^h += ds x_u,
// dL/dw~_dst^h += (sum_u ds) x_v, and dW^h += g^h Z^hT (SNP: g scaled by the merge
// weight of the owner's partial); finally dW += a (x) dL/dw~ and da += W dL/dw~.
#include <algorithm>
#include <vector>

#include "common.cuh"
#include "trainer.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what);
FeatView feat_view(const apt_fstore* f, int r);
apt_status shuffle_items(apt_trainer* t, bool zero_h);
apt_status resample_items(apt_trainer* t, RankState& rs);
apt_status launch_colsum2(apt_ctx* c, const void* g, bool bf16, int64_t pitch, int dim, const int32_t* n_dev,
                          float* out);
}  // namespace apt

#define CK(ctx, expr)                                        \
  do {                                                       \
    apt_status _s = ::apt::check_cuda((ctx), (expr), #expr); \
    if (_s != APT_OK) return _s;                             \
  } while (0)

namespace apt {

constexpr float kSlope = 0.2f;     // LeakyReLU slope of GAT [45]

__device__ __align__(16) uint4 g_gat_zero_row[64];

static int64_t gridn(int64_t n, int t = 256) { return grid_cap(ceil_div(n, t), 16); }

struct GatItems {
  const int32_t* n;       // device item count
  const int32_t* rank;    // requester rank (null: self)
  const int32_t* row;     // requester row (null: the item index)
  const int32_t* gid;     // destination node id
  const int32_t* cnt;     // sampled ELL
  const int32_t* nbr;
  int k;
  int self;
};

struct GatKArgs {
  GatItems it;
  FeatView fv;
  int64_t row_bytes;
  int cols, cpad;         // aggregated columns; lane-padded width (V * EPV)
  int mode;               // 0 full, 1 NFP partial dots into the table, 2 NFP dots read from the table
  int snp_rank;           // >= 0: keep only sources u with part[u] == snp_rank
  const int32_t* part;
  float* const* tab;      // NFP score (fwd) / dalpha (bwd) sums of the requesters: [row][k][H]
  // forward
  const float* wt;        // [2][H][cols]
  float* esc;             // [icap*k][H]
  float* Lm;              // [icap][H]
  float* Ss;              // [icap][H] (SNP)
  void* Z; int z_bf16; int64_t zp;
  float* const* slot_tab; int64_t slot_pitch; int d_out; int C;
  // backward
  const float* gam;       // [icap][H][gp]
  int64_t gp;
  const float* tb;        // [icap][H]
  const float* Lb;        // [icap][H]
  float* dwt;             // [2][H][cols]
};

__device__ __forceinline__ const char* gat_row(const GatKArgs& a, int u) {
  if (a.fv.loc) {
    const int2 l = __ldg(a.fv.loc + u);
    return reinterpret_cast<const char*>(a.fv.base[l.x]) + int64_t(l.y) * a.row_bytes;
  }
  return reinterpret_cast<const char*>(a.fv.base[0]) + int64_t(u) * a.row_bytes;
}

template <int EPV>
__device__ __forceinline__ void unpack(uint4 r, float* x) {
  if constexpr (EPV == 8) {
    x[0] = bf16_lo(r.x); x[1] = bf16_hi(r.x); x[2] = bf16_lo(r.y); x[3] = bf16_hi(r.y);
    x[4] = bf16_lo(r.z); x[5] = bf16_hi(r.z); x[6] = bf16_lo(r.w); x[7] = bf16_hi(r.w);
  } else {
    x[0] = __uint_as_float(r.x); x[1] = __uint_as_float(r.y); x[2] = __uint_as_float(r.z); x[3] = __uint_as_float(r.w);
  }
}

template <int LG>
__device__ __forceinline__ float gsum(float v) {
#pragma unroll
  for (int o = LG / 2; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Fused gather + attention + per-head weighted sums over the owner's items.  A lane
// group of LG lanes owns an item; lane l holds the l-th 16-byte vector of each row.
template <int EPV, int LG, int H>
__global__ void __launch_bounds__(256, 2) gat_fwd_kernel(GatKArgs a) {
  APT_PDL_PROLOGUE();
  extern __shared__ float swt[];                     // [2][H][cpad], zero past cols
  for (int t = threadIdx.x; t < 2 * H * a.cpad; t += blockDim.x) {
    const int c = t % a.cpad, r = t / a.cpad;
    swt[t] = c < a.cols ? a.wt[int64_t(r) * a.cols + c] : 0.f;
  }
  __syncthreads();
  const int lane = lane_id();
  const int sub = LG == 16 ? (lane >> 4) : 0;
  const int l = LG == 16 ? (lane & 15) : lane;
  constexpr int RPW = 32 / LG;
  const int V = a.cpad / EPV;
  const int lv = l < V ? l : 0;
  const int64_t n = *a.it.n;
  const int k = a.it.k;
  const float* ws = swt + lv * EPV;                   // lane's slice of w~_src^h at ws[h * cpad]
  const float* wd = swt + H * a.cpad + lv * EPV;      // (lanes past the row reuse slice 0, masked)
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; w * RPW < n; w += nwarps) {
    const int64_t i = w * RPW + sub;
    const bool valid = i < n;
    const int cnt = valid ? a.it.cnt[i] : 0;
    int cmax = cnt;
    if (LG == 16) cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, 16));
    const int v = valid ? a.it.gid[i] : 0;
    const int row = valid ? (a.it.row ? a.it.row[i] : int(i)) : 0;
    const int rk = valid ? (a.it.rank ? a.it.rank[i] : a.it.self) : 0;
    float er[H];
    if (a.mode != 2) {
      float xv[EPV];
      const uint4 raw = valid ? ld_nc_v4(gat_row(a, v) + lv * 16) : make_uint4(0, 0, 0, 0);
      unpack<EPV>(raw, xv);
#pragma unroll
      for (int h = 0; h < H; ++h) {
        float p = 0.f;
#pragma unroll
        for (int q = 0; q < EPV; ++q) p = fmaf(xv[q], wd[h * a.cpad + q], p);
        er[h] = gsum<LG>(l < V ? p : 0.f);
      }
    }
    float m[H], S[H], acc[H][EPV];
#pragma unroll
    for (int h = 0; h < H; ++h) {
      m[h] = -INFINITY;
      S[h] = 0.f;
#pragma unroll
      for (int q = 0; q < EPV; ++q) acc[h][q] = 0.f;
    }
    for (int e0 = 0; e0 < cmax; e0 += LG) {
      int u = -1;
      if (valid && e0 + l < cnt) u = a.it.nbr[i * k + e0 + l];
      const bool keep = u >= 0 && (a.snp_rank < 0 || a.part[u] == a.snp_rank);
      const char* rp = keep ? gat_row(a, u) : reinterpret_cast<const char*>(g_gat_zero_row);
      const int mloc = min(LG, cmax - e0);
      constexpr int NB = 4;
      for (int j = 0; j < mloc; j += NB) {
        uint4 raw[NB];
        int kp[NB];
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int src_lane = sub * LG + ((j + q) & (LG - 1));
          const char* r = reinterpret_cast<const char*>(__shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(rp), src_lane));
          kp[q] = __shfl_sync(0xffffffffu, int(keep), src_lane) && (j + q < mloc);
          raw[q] = ld_nc_v4(r + lv * 16);
        }
        // phase 1: the NB edges' scores (independent reductions: the shuffles overlap)
        float sc[NB][H];
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int e = e0 + j + q;
          if (a.mode == 2) {
#pragma unroll
            for (int h = 0; h < H; ++h) sc[q][h] = kp[q] ? a.tab[rk][(int64_t(row) * k + e) * H + h] : 0.f;
          } else {
            float xu[EPV];
            unpack<EPV>(raw[q], xu);
#pragma unroll
            for (int h = 0; h < H; ++h) {
              float p = 0.f;
#pragma unroll
              for (int qq = 0; qq < EPV; ++qq) p = fmaf(xu[qq], ws[h * a.cpad + qq], p);
              sc[q][h] = l < V ? p : 0.f;
            }
          }
        }
        if (a.mode != 2) {
#pragma unroll
          for (int o = LG / 2; o > 0; o >>= 1)
#pragma unroll
            for (int q = 0; q < NB; ++q)
#pragma unroll
              for (int h = 0; h < H; ++h) sc[q][h] += __shfl_xor_sync(0xffffffffu, sc[q][h], o);
#pragma unroll
          for (int q = 0; q < NB; ++q)
#pragma unroll
            for (int h = 0; h < H; ++h) sc[q][h] += er[h];
        }
        // phase 2: the online-softmax updates, in edge order
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int e = e0 + j + q;
          float xu[EPV];
          unpack<EPV>(raw[q], xu);
          float s[H];
#pragma unroll
          for (int h = 0; h < H; ++h) s[h] = sc[q][h];
          if (a.mode == 1) {
            if (kp[q] && l < H) {
              float sv = s[0];
#pragma unroll
              for (int h = 1; h < H; ++h) if (l == h) sv = s[h];
              atomicAdd(a.tab[rk] + (int64_t(row) * k + e) * H + l, sv);
            }
            continue;
          }
          if (!kp[q]) continue;
#pragma unroll
          for (int h = 0; h < H; ++h) {
            const float ev = s[h] > 0.f ? s[h] : kSlope * s[h];
            if (l == 0) a.esc[(i * k + e) * H + h] = ev;
            if (ev > m[h]) {            // new running max (uniform in the lane group): rescale once
              const float sc = __expf(m[h] - ev);
              S[h] *= sc;
#pragma unroll
              for (int qq = 0; qq < EPV; ++qq) acc[h][qq] *= sc;
              m[h] = ev;
            }
            const float p = __expf(ev - m[h]);
            S[h] += p;
#pragma unroll
            for (int qq = 0; qq < EPV; ++qq) acc[h][qq] = fmaf(p, xu[qq], acc[h][qq]);
          }
        }
      }
    }
    if (!valid || a.mode == 1) continue;
    // Z^h = acc^h / S^h (the softmax-weighted mean; 0 for an empty row, G3)
#pragma unroll
    for (int h = 0; h < H; ++h) {
      const float inv = S[h] > 0.f ? 1.f / S[h] : 0.f;
      if (l < V) {
        const int64_t o = (i * H + h) * a.zp + l * EPV;
        if (a.z_bf16) {
          uint16_t* z = static_cast<uint16_t*>(a.Z) + o;
          if constexpr (EPV == 8) {   // the lane's 8 columns as one 16-byte store
            *reinterpret_cast<uint4*>(z) =
                make_uint4(pack_bf16x2(acc[h][0] * inv, acc[h][1] * inv), pack_bf16x2(acc[h][2] * inv, acc[h][3] * inv),
                           pack_bf16x2(acc[h][4] * inv, acc[h][5] * inv), pack_bf16x2(acc[h][6] * inv, acc[h][7] * inv));
          } else {
#pragma unroll
            for (int qq = 0; qq < EPV; qq += 2)
              *reinterpret_cast<uint32_t*>(z + qq) = pack_bf16x2(acc[h][qq] * inv, acc[h][qq + 1] * inv);
          }
        } else {
          float* z = static_cast<float*>(a.Z) + o;
#pragma unroll
          for (int qq = 0; qq < EPV; ++qq) z[qq] = acc[h][qq] * inv;
        }
      }
      if (l == 0) {
        if (a.snp_rank >= 0) {
          a.Lm[i * H + h] = m[h];
          a.Ss[i * H + h] = S[h];
          float* sl = a.slot_tab[rk] + (int64_t(row) * a.C + a.it.self) * a.slot_pitch + a.d_out;
          sl[h] = m[h];
          sl[H + h] = S[h];
        } else {
          a.Lm[i * H + h] = S[h] > 0.f ? m[h] + logf(S[h]) : 0.f;
        }
      }
    }
  }
}

// Backward over the owner's items: dalpha, softmax and LeakyReLU backward, and the
// gradients of the two score vectors w~ (accumulated in shared memory per block).
template <int EPV, int LG, int H>
__global__ void __launch_bounds__(256, 2) gat_bwd_kernel(GatKArgs a) {
  APT_PDL_PROLOGUE();
  extern __shared__ float sdw[];                     // [2][H][cpad]
  for (int t = threadIdx.x; t < 2 * H * a.cpad; t += blockDim.x) sdw[t] = 0.f;
  __syncthreads();
  const int lane = lane_id();
  const int sub = LG == 16 ? (lane >> 4) : 0;
  const int l = LG == 16 ? (lane & 15) : lane;
  constexpr int RPW = 32 / LG;
  const int V = a.cpad / EPV;
  const int lv = l < V ? l : 0;
  const int64_t n = *a.it.n;
  const int k = a.it.k;
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  // d w~_src accumulates in registers over every item the lane touches (the lane always
  // owns the same feature columns) and reaches shared memory once per warp at the end;
  // the destination term (one row per item) is combined across the two half-warps first
  float dws[H][EPV];
#pragma unroll
  for (int h = 0; h < H; ++h)
#pragma unroll
    for (int q = 0; q < EPV; ++q) dws[h][q] = 0.f;
  for (int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; w * RPW < n; w += nwarps) {
    const int64_t i = w * RPW + sub;
    const bool valid = i < n;
    const int cnt = valid ? a.it.cnt[i] : 0;
    int cmax = cnt;
    if (LG == 16) cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, 16));
    const int v = valid ? a.it.gid[i] : 0;
    const int row = valid ? (a.it.row ? a.it.row[i] : int(i)) : 0;
    const int rk = valid ? (a.it.rank ? a.it.rank[i] : a.it.self) : 0;
    float gm[H][EPV], t[H], Lv[H], der[H];
#pragma unroll
    for (int h = 0; h < H; ++h) {
#pragma unroll
      for (int q = 0; q < EPV; ++q) {
        const int c = l * EPV + q;
        gm[h][q] = (valid && a.mode != 2 && l < V && c < a.cols) ? a.gam[(i * H + h) * a.gp + c] : 0.f;
      }
      t[h] = valid ? a.tb[i * H + h] : 0.f;
      Lv[h] = valid ? a.Lb[i * H + h] : 0.f;
      der[h] = 0.f;
    }
    for (int e0 = 0; e0 < cmax; e0 += LG) {
      int u = -1;
      if (valid && e0 + l < cnt) u = a.it.nbr[i * k + e0 + l];
      const bool keep = u >= 0 && (a.snp_rank < 0 || a.part[u] == a.snp_rank);
      const char* rp = keep ? gat_row(a, u) : reinterpret_cast<const char*>(g_gat_zero_row);
      const int mloc = min(LG, cmax - e0);
      constexpr int NB = 2;             // (4: register spills at 2 blocks/SM)
      for (int j = 0; j < mloc; j += NB) {
        uint4 raw[NB];
        int kp[NB];
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int src_lane = sub * LG + ((j + q) & (LG - 1));
          const char* r = reinterpret_cast<const char*>(__shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(rp), src_lane));
          kp[q] = __shfl_sync(0xffffffffu, int(keep), src_lane) && (j + q < mloc);
          raw[q] = ld_nc_v4(r + lv * 16);
        }
        float dq[NB][H];     // phase 1: the NB edges' dalpha (independent reductions)
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int e = e0 + j + q;
          if (a.mode == 2) {
#pragma unroll
            for (int h = 0; h < H; ++h) dq[q][h] = kp[q] ? a.tab[rk][(int64_t(row) * k + e) * H + h] : 0.f;
          } else {
            float xu[EPV];
            unpack<EPV>(raw[q], xu);
#pragma unroll
            for (int h = 0; h < H; ++h) {
              float p = 0.f;
#pragma unroll
              for (int qq = 0; qq < EPV; ++qq) p = fmaf(xu[qq], gm[h][qq], p);
              dq[q][h] = p;
            }
          }
        }
        if (a.mode != 2) {
#pragma unroll
          for (int o = LG / 2; o > 0; o >>= 1)
#pragma unroll
            for (int q = 0; q < NB; ++q)
#pragma unroll
              for (int h = 0; h < H; ++h) dq[q][h] += __shfl_xor_sync(0xffffffffu, dq[q][h], o);
        }
#pragma unroll
        for (int q = 0; q < NB; ++q) {
          const int e = e0 + j + q;
          float xu[EPV];
          unpack<EPV>(raw[q], xu);
          float da[H];
#pragma unroll
          for (int h = 0; h < H; ++h) da[h] = dq[q][h];
          if (a.mode == 1) {
            if (kp[q] && l < H) {
              float dv = da[0];
#pragma unroll
              for (int h = 1; h < H; ++h) if (l == h) dv = da[h];
              atomicAdd(a.tab[rk] + (int64_t(row) * k + e) * H + l, dv);
            }
            continue;
          }
          if (!kp[q]) continue;
#pragma unroll
          for (int h = 0; h < H; ++h) {
            const float ev = a.esc[(i * k + e) * H + h];
            const float al = __expf(ev - Lv[h]);
            const float ds = al * (da[h] - t[h]) * (ev > 0.f ? 1.f : kSlope);
            der[h] += ds;
#pragma unroll
            for (int qq = 0; qq < EPV; ++qq) dws[h][qq] = fmaf(ds, xu[qq], dws[h][qq]);
          }
        }
      }
    }
    if (a.mode == 1) continue;                                   // uniform
    float xv[EPV];
    unpack<EPV>(valid ? ld_nc_v4(gat_row(a, v) + lv * 16) : make_uint4(0, 0, 0, 0), xv);
#pragma unroll
    for (int h = 0; h < H; ++h)
#pragma unroll
      for (int q = 0; q < EPV; ++q) {
        float dd = valid ? der[h] * xv[q] : 0.f;
        if (LG == 16) dd += __shfl_xor_sync(0xffffffffu, dd, 16);   // the warp's two items, same columns
        if (sub == 0 && l < V && dd != 0.f) atomicAdd(&sdw[(H + h) * a.cpad + l * EPV + q], dd);
      }
  }
  if (a.mode != 1) {
#pragma unroll
    for (int h = 0; h < H; ++h)
#pragma unroll
      for (int q = 0; q < EPV; ++q) {
        float v = dws[h][q];
        if (LG == 16) v += __shfl_xor_sync(0xffffffffu, v, 16);
        if (sub == 0 && l < V && v != 0.f) atomicAdd(&sdw[h * a.cpad + l * EPV + q], v);
      }
  }
  __syncthreads();
  if (a.mode == 1) return;
  for (int t = threadIdx.x; t < 2 * H * a.cpad; t += blockDim.x) {
    const int c = t % a.cpad, r = t / a.cpad;
    if (c < a.cols && sdw[t] != 0.f) atomicAdd(a.dwt + int64_t(r) * a.cols + c, sdw[t]);
  }
}

// w~_src^h = W^hT a_src^h and w~_dst^h = W^hT a_dst^h over the rank's columns.
__global__ void gat_wt_kernel(const float* __restrict__ W, int64_t ldw, const float* __restrict__ as,
                              const float* __restrict__ ad, int H, int F, int cols, float* __restrict__ wt) {
  APT_PDL_PROLOGUE();
  const int total = 2 * H * cols;
  for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < total; t += gridDim.x * blockDim.x) {
    const int c = t % cols, h = (t / cols) % H, which = t / (cols * H);
    const float* __restrict__ a = (which ? ad : as) + h * F;
    const float* __restrict__ w = W + int64_t(h * F) * ldw + c;
    // independent partial sums: the F row loads of W are in flight together (a chain of
    // F dependent FMAs made this tiny kernel a 20-us latency chain)
    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
    int f = 0;
    for (; f + 4 <= F; f += 4) {
      s0 = fmaf(__ldg(a + f), __ldg(w + int64_t(f) * ldw), s0);
      s1 = fmaf(__ldg(a + f + 1), __ldg(w + int64_t(f + 1) * ldw), s1);
      s2 = fmaf(__ldg(a + f + 2), __ldg(w + int64_t(f + 2) * ldw), s2);
      s3 = fmaf(__ldg(a + f + 3), __ldg(w + int64_t(f + 3) * ldw), s3);
    }
    for (; f < F; ++f) s0 = fmaf(__ldg(a + f), __ldg(w + int64_t(f) * ldw), s0);
    wt[t] = (s0 + s1) + (s2 + s3);
  }
}

// SNP requester: merge the owners' partial (Q_c, m_c, S_c) of every row (online
// softmax combine), + bias, activation; keep the merged log-sum-exp; clear S_c.
__global__ void gat_snp_merge_kernel(float* __restrict__ slot, int64_t sp, int C, int H, int F,
                                     const int32_t* __restrict__ n_p, const float* __restrict__ b, int relu,
                                     float* __restrict__ Hout, int64_t h_pitch, float* __restrict__ Lr) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int d_out = H * F;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < n * H; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / H;
    const int h = int(t - r * H);
    float* base = slot + r * C * sp;
    float m = -INFINITY;
    for (int c = 0; c < C; ++c) {
      const float* s = base + c * sp + d_out;
      if (s[H + h] > 0.f) m = fmaxf(m, s[h]);
    }
    float wsum = 0.f;
    float w[kMaxRanks];
    for (int c = 0; c < C; ++c) {
      const float* s = base + c * sp + d_out;
      w[c] = s[H + h] > 0.f ? s[H + h] * expf(s[h] - m) : 0.f;
      wsum += w[c];
    }
    const float inv = wsum > 0.f ? 1.f / wsum : 0.f;
    for (int f = 0; f < F; ++f) {
      float acc = 0.f;
      for (int c = 0; c < C; ++c)
        if (w[c] > 0.f) acc = fmaf(w[c], base[c * sp + h * F + f], acc);
      float o = acc * inv + b[h * F + f];
      Hout[r * h_pitch + h * F + f] = relu ? fmaxf(o, 0.f) : o;
    }
    Lr[r * H + h] = wsum > 0.f ? m + logf(wsum) : 0.f;
    for (int c = 0; c < C; ++c) base[c * sp + d_out + H + h] = 0.f;   // self-cleaning for the next step
  }
}

// Requester: t^h = sum_f g[hF+f] (h1[hF+f] - b[hF+f]) -- g . (pre - b): with a ReLU
// g is already 0 where h1 = 0, elsewhere h1 = pre.
template <typename T>
__global__ void gat_t_kernel(const T* __restrict__ g, int64_t gp, const float* __restrict__ h1, int64_t hp,
                             const float* __restrict__ b, int H, int F, const int32_t* __restrict__ n_p,
                             float* __restrict__ t) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int lane = lane_id();
  const int64_t nw = int64_t(gridDim.x) * (blockDim.x >> 5);
  if constexpr (sizeof(T) == 2) {
    if (F % 8 == 0 && gp % 8 == 0 && hp % 4 == 0 && H <= 8) {
      // 8 columns of one head per lane and chunk: 16-byte g loads, 2 x 16-byte h loads
      const int nv = H * F / 8;
      for (int64_t r = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; r < n; r += nw) {
        float s[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
        for (int v = lane; v < nv; v += 32) {
          const int c = v * 8, h = c / F;
          const uint4 gr = *reinterpret_cast<const uint4*>(g + r * gp + c);
          const float4 h0 = *reinterpret_cast<const float4*>(h1 + r * hp + c);
          const float4 h4 = *reinterpret_cast<const float4*>(h1 + r * hp + c + 4);
          const float4 b0 = *reinterpret_cast<const float4*>(b + c);
          const float4 b4 = *reinterpret_cast<const float4*>(b + c + 4);
          float acc = 0.f;
          acc = fmaf(bf16_lo(gr.x), h0.x - b0.x, acc); acc = fmaf(bf16_hi(gr.x), h0.y - b0.y, acc);
          acc = fmaf(bf16_lo(gr.y), h0.z - b0.z, acc); acc = fmaf(bf16_hi(gr.y), h0.w - b0.w, acc);
          acc = fmaf(bf16_lo(gr.z), h4.x - b4.x, acc); acc = fmaf(bf16_hi(gr.z), h4.y - b4.y, acc);
          acc = fmaf(bf16_lo(gr.w), h4.z - b4.z, acc); acc = fmaf(bf16_hi(gr.w), h4.w - b4.w, acc);
#pragma unroll
          for (int q = 0; q < 8; ++q) if (q == h) s[q] += acc;
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          if (q >= H) break;
          const float tot = warp_sum(s[q]);
          if (lane == 0) t[r * H + q] = tot;
        }
      }
      return;
    }
  }
  for (int64_t r = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; r < n; r += nw) {   // warp per row
    for (int h = 0; h < H; ++h) {
      float s = 0.f;
      for (int f = lane; f < F; f += 32) {
        const int c = h * F + f;
        float gv;
        if constexpr (sizeof(T) == 2) gv = __uint_as_float(uint32_t(g[r * gp + c]) << 16);
        else gv = float(g[r * gp + c]);
        s = fmaf(gv, h1[r * hp + c] - b[c], s);
      }
      s = warp_sum(s);
      if (lane == 0) t[r * H + h] = s;
    }
  }
}

// Owner: g rows (fp32), t and the global log-sum-exp of its items from the
// requesters; SNP scales g by the merge weight omega_c = S_c e^{m_c - L}.
// bf16 mode (T = uint16_t) writes the bf16 operands of the tcgen05 contractions and zeroes
// their rows [n, round_up(n, 64)) (the weight-gradient kernel's row-block tail).
template <typename T>
__global__ void gat_gather_kernel(T* const* __restrict__ gtab, int64_t gp, float* const* __restrict__ ttab,
                                  float* const* __restrict__ Ltab, GatItems it, int H, int F,
                                  const float* __restrict__ Lm, const float* __restrict__ Ss, int snp,
                                  float* __restrict__ wG, float* __restrict__ wGs, int64_t wp,
                                  uint16_t* __restrict__ wGb, uint16_t* __restrict__ wGsb, int64_t wpb, int64_t icap,
                                  float* __restrict__ tb, float* __restrict__ Lb) {
  APT_PDL_PROLOGUE();
  const int64_t n = *it.n;
  const int64_t rows = sizeof(T) == 2 ? std::min<int64_t>(icap, round_up(n, 64)) : n;
  const int d_out = H * F;
  if constexpr (sizeof(T) == 2) {
    if (F % 8 == 0 && gp % 8 == 0 && wpb % 8 == 0) {
      // bf16 rows in 16-byte vectors (8 columns of one head per thread)
      const int nv = d_out / 8;
      for (int64_t x = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < rows * nv; x += int64_t(gridDim.x) * blockDim.x) {
        const int64_t i = x / nv;
        const int c = int(x - i * nv) * 8;
        uint4* dst = reinterpret_cast<uint4*>(wGb + i * wpb + c);
        uint4* dsts = snp ? reinterpret_cast<uint4*>(wGsb + i * wpb + c) : nullptr;
        if (i >= n) {
          *dst = make_uint4(0, 0, 0, 0);
          if (dsts) *dsts = make_uint4(0, 0, 0, 0);
          continue;
        }
        const int h = c / F;
        const int rk = it.rank ? it.rank[i] : it.self;
        const int row = it.row ? it.row[i] : int(i);
        const uint4 graw = *reinterpret_cast<const uint4*>(gtab[rk] + int64_t(row) * gp + c);
        *dst = graw;
        const float L = snp ? Ltab[rk][int64_t(row) * H + h] : Lm[i * H + h];
        if (dsts) {
          const float om = Ss[i * H + h] > 0.f ? Ss[i * H + h] * expf(Lm[i * H + h] - L) : 0.f;
          const uint32_t w4[4] = {graw.x, graw.y, graw.z, graw.w};
          uint32_t o4[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) o4[q] = pack_bf16x2(bf16_lo(w4[q]) * om, bf16_hi(w4[q]) * om);
          *dsts = make_uint4(o4[0], o4[1], o4[2], o4[3]);
        }
        if (c % F == 0) {
          tb[i * H + h] = ttab[rk][int64_t(row) * H + h];
          Lb[i * H + h] = L;
        }
      }
      return;
    }
  }
  for (int64_t x = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; x < rows * d_out; x += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = x / d_out;
    const int c = int(x - i * d_out);
    if (i >= n) {
      wGb[i * wpb + c] = 0;
      if (snp) wGsb[i * wpb + c] = 0;
      continue;
    }
    const int h = c / F;
    const int rk = it.rank ? it.rank[i] : it.self;
    const int row = it.row ? it.row[i] : int(i);
    const T graw = gtab[rk][int64_t(row) * gp + c];
    float gv;
    if constexpr (sizeof(T) == 2) gv = __uint_as_float(uint32_t(graw) << 16);
    else gv = float(graw);
    const float L = snp ? Ltab[rk][int64_t(row) * H + h] : Lm[i * H + h];
    const float om = snp ? (Ss[i * H + h] > 0.f ? Ss[i * H + h] * expf(Lm[i * H + h] - L) : 0.f) : 1.f;
    if constexpr (sizeof(T) == 2) {
      wGb[i * wpb + c] = graw;
      if (snp) {
        __nv_bfloat16 q = __float2bfloat16_rn(gv * om);
        wGsb[i * wpb + c] = *reinterpret_cast<uint16_t*>(&q);
      }
    } else {
      wG[i * wp + c] = gv;
      if (snp) wGs[i * wp + c] = gv * om;
    }
    if (c % F == 0) {
      tb[i * H + h] = ttab[rk][int64_t(row) * H + h];
      Lb[i * H + h] = L;
    }
  }
}

// dW[hF+f][c] += a_src[hF+f] dw~_src^h[c] + a_dst[hF+f] dw~_dst^h[c];
// da_src[hF+f] += sum_c W[hF+f][c] dw~_src^h[c] (and dst).  One block per output row.
__global__ void gat_fold_kernel(const float* __restrict__ W, int64_t ldw, const float* __restrict__ as,
                                const float* __restrict__ ad, const float* __restrict__ dwt, int H, int F, int cols,
                                float* __restrict__ dW, int64_t lddw, float* __restrict__ das, float* __restrict__ dad) {
  APT_PDL_PROLOGUE();
  __shared__ float red[2][256];
  const int o = blockIdx.x;           // output row hF + f
  const int h = o / F;
  const float* gs = dwt + int64_t(h) * cols;
  const float* gd = dwt + int64_t(H + h) * cols;
  float s0 = 0.f, s1 = 0.f;
  for (int c = threadIdx.x; c < cols; c += blockDim.x) {
    dW[int64_t(o) * lddw + c] += as[o] * gs[c] + ad[o] * gd[c];
    const float w = W[int64_t(o) * ldw + c];
    s0 = fmaf(w, gs[c], s0);
    s1 = fmaf(w, gd[c], s1);
  }
  red[0][threadIdx.x] = s0;
  red[1][threadIdx.x] = s1;
  __syncthreads();
  for (int st = blockDim.x / 2; st > 0; st >>= 1) {
    if (threadIdx.x < st) {
      red[0][threadIdx.x] += red[0][threadIdx.x + st];
      red[1][threadIdx.x] += red[1][threadIdx.x + st];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    das[o] += red[0][0];
    dad[o] += red[1][0];
  }
}

__global__ void gat_bias_act_kernel(float* __restrict__ Hb, int64_t pitch, int dim, const float* __restrict__ b,
                                    int relu, const int32_t* __restrict__ n_p) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < n * dim; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / dim;
    const int c = int(t - r * dim);
    const float v = Hb[r * pitch + c] + b[c];
    Hb[r * pitch + c] = relu ? fmaxf(v, 0.f) : v;
  }
}

// ------------------------------------------------------------------ host side
static bool gdp_path(const apt_trainer* t) { return t->world == 1 || t->s == APT_GDP; }

static GatItems items_of(apt_trainer* t, RankState& rs) {
  const Hop& hp = rs.hops[t->K - 1];
  if (gdp_path(t)) return GatItems{hp.n_dst, nullptr, nullptr, hp.dst, hp.cnt, hp.nbr, hp.k, rs.rank};
  const Xchg& x = rs.x;
  return GatItems{x.n_work, x.work_rank, x.work_row, x.work_gid, x.wcnt, x.wnbr, hp.k, rs.rank};
}

// W^1 as the rank uses it: fp32 master (scores, w~) and the projection operand
// (bf16 copy in bf16 mode), full or the NFP column slice.
struct WView { const float* Wf; int64_t ldf; const void* Wp; DType wt; int64_t ldp; float* dW; int64_t lddw; };
static WView wview(apt_trainer* t, RankState& rs) {
  const Layer& L = rs.L[0];
  const bool bf = t->m.dtype == APT_BF16;
  if (rs.x.W1s) {
    const int w = std::max(rs.x.w_cols, 1);
    return WView{rs.x.W1s, w, bf ? static_cast<const void*>(rs.x.Wb1s) : rs.x.W1s, bf ? kBF16 : kF32,
                 bf ? rs.x.ws_pitch : w, rs.x.dW1s, w};
  }
  return WView{L.W, L.d_in, bf ? static_cast<const void*>(L.Wb) : L.W, bf ? kBF16 : kF32, bf ? L.wb_pitch : L.d_in,
               L.dW, L.d_in};
}

static GatKArgs kargs(apt_trainer* t, RankState& rs) {
  GatState& ga = rs.ga;
  GatKArgs a{};
  a.it = items_of(t, rs);
  a.fv = feat_view(t->f, rs.rank);
  a.row_bytes = a.fv.pitch * (a.fv.dtype == kBF16 ? 2 : 4);
  a.cols = ga.cols;
  const int epv = a.fv.dtype == kBF16 ? 8 : 4;
  a.cpad = int(round_up(ga.cols, epv));
  a.snp_rank = (t->s == APT_SNP && !gdp_path(t)) ? rs.rank : -1;
  a.part = t->g->part;
  a.wt = ga.wt;
  a.esc = ga.esc;
  a.Lm = ga.Lm;
  a.Ss = ga.Ss;
  a.Z = ga.Z;
  a.z_bf16 = t->m.dtype == APT_BF16;
  a.zp = ga.zp;
  a.slot_tab = t->slot_tab;
  a.slot_pitch = rs.ga.slot_pitch;
  a.d_out = rs.L[0].d_out;
  a.C = t->world;
  a.gam = ga.Gam;
  a.gp = ga.gp;
  a.tb = ga.tb;
  a.Lb = ga.Lb;
  a.dwt = ga.dwt;
  return a;
}

template <int EPV, int LG, int H>
static cudaError_t launch_one(const GatKArgs& a, bool bwd, int64_t max_items, cudaStream_t st) {
  constexpr int RPW = 32 / LG;
  const int64_t blocks = grid_cap(ceil_div(ceil_div(max_items, RPW) * 32, 256), 8);
  const size_t smem = size_t(2) * H * a.cpad * sizeof(float);
  if (bwd) return launch_pdl(gat_bwd_kernel<EPV, LG, H>, dim3(blocks), dim3(256), smem, st, a);
  return launch_pdl(gat_fwd_kernel<EPV, LG, H>, dim3(blocks), dim3(256), smem, st, a);
}

template <int EPV, int LG>
static cudaError_t launch_h(const GatKArgs& a, bool bwd, int H, int64_t mi, cudaStream_t st) {
  switch (H) {
    case 1: return launch_one<EPV, LG, 1>(a, bwd, mi, st);
    case 2: return launch_one<EPV, LG, 2>(a, bwd, mi, st);
    case 4: return launch_one<EPV, LG, 4>(a, bwd, mi, st);
    case 8: return launch_one<EPV, LG, 8>(a, bwd, mi, st);
    default: return cudaErrorInvalidValue;
  }
}

static apt_status launch_gat(apt_trainer* t, const GatKArgs& a, bool bwd, int64_t max_items) {
  apt_ctx* c = t->ctx;
  const bool bf = a.fv.dtype == kBF16;
  const int V = a.cpad / (bf ? 8 : 4);
  if (V > 32) return set_err(c, APT_E_UNSUPPORTED, "GAT layer: %d feature columns exceed one warp's row", a.cols);
  const int H = t->gat_heads;
  cudaError_t e;
  if (bf) e = V <= 16 ? launch_h<8, 16>(a, bwd, H, max_items, c->stream) : launch_h<8, 32>(a, bwd, H, max_items, c->stream);
  else e = V <= 16 ? launch_h<4, 16>(a, bwd, H, max_items, c->stream) : launch_h<4, 32>(a, bwd, H, max_items, c->stream);
  CK(c, e);
  c->launches++;
  return APT_OK;
}

template <typename T>
static T* upload(apt_trainer* t, const std::vector<T>& v) {
  T* d = t->arena.alloc<T>(int64_t(v.size()), false);
  if (d) cudaMemcpyAsync(d, v.data(), sizeof(T) * v.size(), cudaMemcpyHostToDevice, t->ctx->stream);
  return d;
}

apt_status gat_alloc(apt_trainer* t, RankState& rs) {
  apt_ctx* c = t->ctx;
  Arena& A = t->arena;
  GatState& ga = rs.ga;
  const Layer& L = rs.L[0];
  const Hop& hp = rs.hops[t->K - 1];
  const int C = t->world;
  const bool gdp = gdp_path(t);
  ga.H = t->gat_heads;
  ga.F = L.d_out / ga.H;
  ga.cols = (!gdp && rs.x.W1s) ? rs.x.w_cols : L.d_in;
  ga.zp = round_up(std::max(ga.cols, 1), 8);
  ga.icap = gdp ? hp.max_dst : rs.x.wcap;
  const int64_t H = ga.H, ic = ga.icap, wp = round_up(L.d_out, 4);
  const size_t esz = t->m.dtype == APT_BF16 ? 2 : 4;
  ga.a_src = A.alloc<float>(L.d_out, true);
  ga.a_dst = A.alloc<float>(L.d_out, true);
  ga.wt = A.alloc<float>(2 * H * std::max(ga.cols, 1), true);
  ga.dwt = A.alloc<float>(2 * H * std::max(ga.cols, 1), true);
  ga.Z = A.alloc<uint8_t>(int64_t(ic * H * ga.zp * esz), true);
  ga.esc = A.alloc<float>(ic * hp.k * H, false);
  ga.Lm = A.alloc<float>(ic * H, true);
  ga.Ss = A.alloc<float>(ic * H, true);
  ga.Lb = A.alloc<float>(ic * H, true);
  ga.tb = A.alloc<float>(ic * H, true);
  const bool snp = t->s == APT_SNP && !gdp;
  if (esz == 2) {
    ga.wpb = round_up(L.d_out, 8);
    ga.wGb = A.alloc<uint16_t>(ic * ga.wpb, true);
    ga.wGsb = snp ? A.alloc<uint16_t>(ic * ga.wpb, true) : ga.wGb;
    ga.wG = ga.wGs = reinterpret_cast<float*>(ga.wGb);   // (unused in bf16 mode; non-null marker)
  } else {
    ga.wG = A.alloc<float>(ic * wp, true);
    ga.wGs = snp ? A.alloc<float>(ic * wp, true) : ga.wG;
  }
  ga.gp = round_up(std::max(ga.cols, 1), 4);
  ga.Gam = A.alloc<float>(ic * H * ga.gp, true);
  ga.t = A.alloc<float>(L.max_rows * H, true);
  if (!gdp && t->s == APT_SNP) {
    ga.slot_pitch = round_up(L.d_out + 2 * H, 4);
    ga.Lr = A.alloc<float>(L.max_rows * H, true);
    ga.slot = A.alloc<float>(L.max_rows * C * ga.slot_pitch, true);
  }
  if (!gdp && t->s == APT_NFP) {
    ga.ssum = A.alloc<float>(L.max_rows * hp.k * H, true);
    ga.dsum = A.alloc<float>(L.max_rows * hp.k * H, true);
  }
  if (!ga.Gam || !ga.wG || !ga.wGs || !ga.esc || !ga.Z || !ga.t || (!gdp && t->s == APT_SNP && !ga.slot) ||
      (!gdp && t->s == APT_NFP && !ga.dsum))
    return set_err(c, APT_E_OOM, "GAT layer: out of device memory (%lld items)", (long long)ic);
  return APT_OK;
}

// Pointer tables over the ranks (peer-mapped in a job of one process per GPU).
apt_status gat_tables(apt_trainer* t) {
  apt_ctx* c = t->ctx;
  const int C = t->world;
  std::vector<float*> tt(C), lr(C), sl(C), ss(C), ds(C), gg(C);
  std::vector<uint16_t*> gb(C);
  if (multiprocess(c)) {
    RankState& rs = t->R[0];
    auto share = [&](auto& tab, auto* mine) -> apt_status {
      if (!mine) return APT_OK;
      std::vector<void*> v(C, nullptr);
      apt_status s = share_ptr(c, mine, v.data(), &t->peer_opened);
      for (int p = 0; p < C; ++p) tab[p] = static_cast<std::remove_reference_t<decltype(tab[0])>>(v[p]);
      return s;
    };
    apt_status s;
    if ((s = share(tt, rs.ga.t)) != APT_OK || (s = share(lr, rs.ga.Lr)) != APT_OK ||
        (s = share(sl, rs.ga.slot)) != APT_OK || (s = share(ss, rs.ga.ssum)) != APT_OK ||
        (s = share(ds, rs.ga.dsum)) != APT_OK || (s = share(gg, rs.L[0].G)) != APT_OK ||
        (s = share(gb, rs.L[0].Gb)) != APT_OK)
      return s;
  } else {
    for (auto& rs : t->R) {
      tt[rs.rank] = rs.ga.t;
      lr[rs.rank] = rs.ga.Lr;
      sl[rs.rank] = rs.ga.slot;
      ss[rs.rank] = rs.ga.ssum;
      ds[rs.rank] = rs.ga.dsum;
      gg[rs.rank] = rs.L[0].G;
      gb[rs.rank] = rs.L[0].Gb;
    }
  }
  t->gt_tab = upload(t, tt);
  t->gL_tab = upload(t, lr);
  t->slot_tab = upload(t, sl);
  t->ssum_tab = upload(t, ss);
  t->dsum_tab = upload(t, ds);
  t->gG_tab = upload(t, gg);
  t->gGb_tab = upload(t, gb);
  if (!gdp_path(t)) {
    for (auto& rs : t->R) {
      GatState& ga = rs.ga;
      std::vector<float*> o(size_t(ga.H) * C, nullptr);
      for (int h = 0; h < ga.H; ++h)
        for (int r = 0; r < C; ++r)
          o[size_t(h) * C + r] = t->s == APT_SNP ? sl[r] + int64_t(rs.rank) * ga.slot_pitch + h * ga.F
                                                 : t->h1_host[r] + h * ga.F;
      ga.otab = upload(t, o);
      if (!ga.otab) return set_err(c, APT_E_OOM, "GAT tables: out of device memory");
    }
  }
  if (!t->gGb_tab) return set_err(c, APT_E_OOM, "GAT tables: out of device memory");
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

// Forward of the GAT first layer for every hosted rank under the trainer's strategy.
apt_status gat_layer1_fwd(apt_trainer* t, bool time_it) {
  apt_ctx* c = t->ctx;
  const bool gdp = gdp_path(t);
  const bool bf = t->m.dtype == APT_BF16;
  const int H = t->gat_heads;
  for (auto& rs : t->R) {
    GatState& ga = rs.ga;
    const WView wv = wview(t, rs);
    launch_pdl(gat_wt_kernel, dim3(gridn(2 * H * std::max(ga.cols, 1))), dim3(256), 0, c->stream, wv.Wf, wv.ldf,
               ga.a_src, ga.a_dst, H, ga.F, ga.cols, ga.wt);
    CK(c, cudaGetLastError());
    c->launches++;
  }
  if (!gdp) {
    if (t->s == APT_NFP)
      for (auto& rs : t->R)
        CK(c, cudaMemsetAsync(rs.ga.ssum, 0, sizeof(float) * rs.L[0].max_rows * rs.hops[t->K - 1].k * H, c->stream));
    apt_status s = shuffle_items(t, t->s == APT_NFP);
    if (s != APT_OK) return s;
    for (auto& rs : t->R)
      if ((s = resample_items(t, rs)) != APT_OK) return s;
  }
  bool first = time_it;
  auto run = [&](RankState& rs, int mode) -> apt_status {
    GatKArgs a = kargs(t, rs);
    a.mode = mode;
    a.tab = t->ssum_tab;
    if (first && mode != 1) CK(c, tap_event(t, t->ev[6], c->stream));
    apt_status s = launch_gat(t, a, false, rs.ga.icap);
    if (s != APT_OK) return s;
    if (first && mode != 1) {
      CK(c, tap_event(t, t->ev[7], c->stream));
      first = false;
    }
    return APT_OK;
  };
  if (!gdp && t->s == APT_NFP) {
    for (auto& rs : t->R) { apt_status s = run(rs, 1); if (s != APT_OK) return s; }
    { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // every partial score summed
    for (auto& rs : t->R) { apt_status s = run(rs, 2); if (s != APT_OK) return s; }
  } else {
    for (auto& rs : t->R) { apt_status s = run(rs, 0); if (s != APT_OK) return s; }
  }
  // projection per head: pre^h = W^h Z^h (routed into the requesters' buffers)
  for (auto& rs : t->R) {
    GatState& ga = rs.ga;
    Layer& L = rs.L[0];
    const WView wv = wview(t, rs);
    const GatItems it = items_of(t, rs);
    const bool tc = bf && ga.F % 4 == 0 && ga.cols > 0 && tc_gemm_supported(ga.F, ga.cols);
    for (int h = 0; h < H && tc; ++h) {   // tcgen05: A = Z^h (K-major, pitch H*zp), B = W^h
      TcGemmArgs g{};
      g.Z = static_cast<const uint16_t*>(ga.Z) + size_t(h) * ga.zp;
      g.z_pitch = int64_t(H) * ga.zp;
      g.W = static_cast<const uint16_t*>(wv.Wp) + size_t(h) * ga.F * wv.ldp;
      g.w_pitch = wv.ldp;
      g.M_max = ga.icap; g.M_dev = it.n; g.N = ga.F; g.K = ga.cols;
      if (gdp) {
        g.Y = L.H + h * ga.F; g.y_pitch = L.h_pitch;
        g.bias = L.b + h * ga.F; g.relu = t->K > 1 ? 1 : 0;
      } else {
        g.out_base = ga.otab + size_t(h) * t->world; g.out_rank = it.rank; g.out_row = it.row;
        if (t->s == APT_SNP) {
          g.y_pitch = int64_t(t->world) * ga.slot_pitch;
        } else {
          g.y_pitch = L.h_pitch;
          if (t->s == APT_DNP) { g.bias = L.b + h * ga.F; g.relu = t->K > 1 ? 1 : 0; }
          else g.accumulate = 1;
        }
      }
      CK(c, launch_tc_gemm(g, c->stream));
      c->launches++;
    }
    for (int h = 0; h < H && !tc; ++h) {
      SimtGemmArgs g{};
      g.A = static_cast<const uint8_t*>(ga.Z) + size_t(h) * ga.zp * (bf ? 2 : 4);
      g.a_t = bf ? kBF16 : kF32;
      g.sam = int64_t(H) * ga.zp;
      g.sak = 1;
      g.B = static_cast<const uint8_t*>(wv.Wp) + size_t(h) * ga.F * wv.ldp * (bf ? 2 : 4);
      g.b_t = wv.wt;
      g.sbk = 1;
      g.sbn = wv.ldp;
      g.M_dev = it.n;
      g.M = ga.icap;
      g.N = ga.F;
      g.K = ga.cols;
      if (gdp) {
        g.C = L.H + h * ga.F;
        g.ldc = L.h_pitch;
        g.bias = L.b + h * ga.F;
        g.relu = t->K > 1 ? 1 : 0;
      } else {
        g.out_base = ga.otab + size_t(h) * t->world;
        g.out_rank = it.rank;
        g.out_row = it.row;
        if (t->s == APT_SNP) {
          g.ldc = int64_t(t->world) * ga.slot_pitch;
        } else {
          g.ldc = L.h_pitch;
          if (t->s == APT_DNP) { g.bias = L.b + h * ga.F; g.relu = t->K > 1 ? 1 : 0; }
          else g.accumulate = 1;
        }
      }
      if (ga.cols > 0) CK(c, launch_simt_gemm(g, c->stream));
      c->launches++;
    }
  }
  if (gdp) return APT_OK;
  { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // every partial / row delivered
  for (auto& rs : t->R) {
    Layer& L = rs.L[0];
    GatState& ga = rs.ga;
    if (t->s == APT_SNP) {
      launch_pdl(gat_snp_merge_kernel, dim3(gridn(L.max_rows * H)), dim3(256), 0, c->stream, ga.slot, ga.slot_pitch,
                 t->world, H, ga.F, L.n_rows, static_cast<const float*>(L.b), t->K > 1 ? 1 : 0, L.H, L.h_pitch, ga.Lr);
    } else if (t->s == APT_NFP) {
      launch_pdl(gat_bias_act_kernel, dim3(gridn(L.max_rows * L.d_out)), dim3(256), 0, c->stream, L.H, L.h_pitch,
                 L.d_out, static_cast<const float*>(L.b), t->K > 1 ? 1 : 0, L.n_rows);
    } else {
      continue;
    }
    CK(c, cudaGetLastError());
    c->launches++;
  }
  return APT_OK;
}

// Backward of the GAT first layer.  On entry every requester's G (fp32 mode) / Gb
// (bf16 mode) holds dL/dpre^1 and the layer-1 gradients (dW^1 or the NFP slice
// dW1s, db^1, da) are zero; on exit they hold this rank's contributions (the
// caller all-reduces).
apt_status gat_layer1_bwd(apt_trainer* t) {
  apt_ctx* c = t->ctx;
  const bool gdp = gdp_path(t);
  const bool bf = t->m.dtype == APT_BF16;
  const int H = t->gat_heads;
  for (auto& rs : t->R) {    // requesters: t = g . (pre - b), db = sum g
    Layer& L = rs.L[0];
    GatState& ga = rs.ga;
    if (bf) launch_pdl(gat_t_kernel<uint16_t>, dim3(gridn(L.max_rows * 32)), dim3(256), 0, c->stream,
                       static_cast<const uint16_t*>(L.Gb), L.gb_pitch, static_cast<const float*>(L.H), L.h_pitch,
                       static_cast<const float*>(L.b), H, ga.F, L.n_rows, ga.t);
    else launch_pdl(gat_t_kernel<float>, dim3(gridn(L.max_rows * 32)), dim3(256), 0, c->stream,
                    static_cast<const float*>(L.G), L.h_pitch, static_cast<const float*>(L.H), L.h_pitch,
                    static_cast<const float*>(L.b), H, ga.F, L.n_rows, ga.t);
    CK(c, cudaGetLastError());
    c->launches++;
    apt_status s = bf ? launch_colsum2(c, L.Gb, true, L.gb_pitch, L.d_out, L.n_rows, L.db)
                      : launch_colsum2(c, L.G, false, L.h_pitch, L.d_out, L.n_rows, L.db);
    if (s != APT_OK) return s;
    if (!gdp && t->s == APT_NFP)
      CK(c, cudaMemsetAsync(ga.dsum, 0, sizeof(float) * L.max_rows * rs.hops[t->K - 1].k * H, c->stream));
  }
  if (!gdp) { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // g, t, merged L ready
  const int64_t wp = round_up(t->R[0].L[0].d_out, 4);
  for (auto& rs : t->R) {    // owners: gather, gamma = W^T g (per head)
    GatState& ga = rs.ga;
    Layer& L = rs.L[0];
    const GatItems it = items_of(t, rs);
    const WView wv = wview(t, rs);
    CK(c, cudaMemsetAsync(ga.dwt, 0, sizeof(float) * 2 * H * std::max(ga.cols, 1), c->stream));
    if (rs.x.W1s && !gdp) CK(c, cudaMemsetAsync(rs.x.dW1s, 0, sizeof(float) * L.d_out * std::max(rs.x.w_cols, 1), c->stream));
    const int snp = (!gdp && t->s == APT_SNP) ? 1 : 0;
    if (bf) launch_pdl(gat_gather_kernel<uint16_t>, dim3(gridn(ga.icap * L.d_out)), dim3(256), 0, c->stream,
                       t->gGb_tab, L.gb_pitch, t->gt_tab, t->gL_tab, it, H, ga.F,
                       static_cast<const float*>(ga.Lm), static_cast<const float*>(ga.Ss), snp,
                       static_cast<float*>(nullptr), static_cast<float*>(nullptr), wp, ga.wGb, ga.wGsb, ga.wpb, ga.icap,
                       ga.tb, ga.Lb);
    else launch_pdl(gat_gather_kernel<float>, dim3(gridn(ga.icap * L.d_out)), dim3(256), 0, c->stream,
                    t->gG_tab, L.h_pitch, t->gt_tab, t->gL_tab, it, H, ga.F,
                    static_cast<const float*>(ga.Lm), static_cast<const float*>(ga.Ss), snp, ga.wG, ga.wGs, wp,
                    static_cast<uint16_t*>(nullptr), static_cast<uint16_t*>(nullptr), int64_t(0), ga.icap, ga.tb, ga.Lb);
    CK(c, cudaGetLastError());
    c->launches++;
    // gamma^h = W^hT g^h: tcgen05 with W read N-major as stored (bf16 mode), else fp32 CUDA cores
    const bool tcg = bf && ga.F % 16 == 0 && ga.cols > 0 && tc_gemm_supported(ga.cols, ga.F);
    for (int h = 0; h < H; ++h) {
      if (tcg) {
        TcGemmArgs g{};
        g.Z = ga.wGb + h * ga.F; g.z_pitch = ga.wpb;
        g.W = static_cast<const uint16_t*>(wv.Wp) + size_t(h) * ga.F * wv.ldp; g.w_pitch = wv.ldp; g.w_mn = 1;
        g.M_max = ga.icap; g.M_dev = it.n; g.N = ga.cols; g.K = ga.F;
        g.Y = ga.Gam + int64_t(h) * ga.gp; g.y_pitch = int64_t(H) * ga.gp;
        CK(c, launch_tc_gemm(g, c->stream));
      } else {
        SimtGemmArgs g{};
        if (bf) { g.A = ga.wGb + h * ga.F; g.a_t = kBF16; g.sam = ga.wpb; }
        else { g.A = ga.wG + h * ga.F; g.a_t = kF32; g.sam = wp; }
        g.sak = 1;
        g.B = static_cast<const uint8_t*>(wv.Wp) + size_t(h) * ga.F * wv.ldp * (bf ? 2 : 4);
        g.b_t = wv.wt; g.sbk = wv.ldp; g.sbn = 1;
        g.C = ga.Gam + int64_t(h) * ga.gp; g.ldc = int64_t(H) * ga.gp;
        g.M_dev = it.n; g.M = ga.icap; g.N = ga.cols; g.K = ga.F;
        if (ga.cols > 0) CK(c, launch_simt_gemm(g, c->stream));
      }
      c->launches++;
    }
    if (!gdp && t->s == APT_NFP) {
      GatKArgs a = kargs(t, rs);
      a.mode = 1;
      a.tab = t->dsum_tab;
      apt_status s = launch_gat(t, a, true, ga.icap);
      if (s != APT_OK) return s;
    }
  }
  if (!gdp && t->s == APT_NFP) { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // dalpha summed
  for (auto& rs : t->R) {    // owners: softmax backward, dw~, dW (projection part), fold
    GatState& ga = rs.ga;
    Layer& L = rs.L[0];
    const GatItems it = items_of(t, rs);
    const WView wv = wview(t, rs);
    GatKArgs a = kargs(t, rs);
    a.mode = (!gdp && t->s == APT_NFP) ? 2 : 0;
    a.tab = t->dsum_tab;
    apt_status s = launch_gat(t, a, true, ga.icap);
    if (s != APT_OK) return s;
    // dW^h += (omega g^h)^T Z^h: tcgen05 weight-gradient kernel (bf16), else fp32 split-K
    const bool tcw = bf && ga.F % 8 == 0 && ga.cols > 0 && tc_wgrad_supported(ga.F, ga.cols);
    for (int h = 0; h < H; ++h) {
      if (tcw) {
        TcWgradArgs w{ga.wGsb + h * ga.F, ga.wpb, static_cast<const uint16_t*>(ga.Z) + size_t(h) * ga.zp,
                      int64_t(H) * ga.zp, it.n, ga.icap, ga.F, ga.cols, wv.dW + int64_t(h) * ga.F * wv.lddw, nullptr,
                      wv.lddw};
        CK(c, launch_tc_wgrad(w, c->stream));
      } else {
        SimtGemmArgs g{};
        if (bf) { g.A = ga.wGsb + h * ga.F; g.a_t = kBF16; g.sak = ga.wpb; }
        else { g.A = ga.wGs + h * ga.F; g.a_t = kF32; g.sak = wp; }
        g.sam = 1;
        g.B = static_cast<const uint8_t*>(ga.Z) + size_t(h) * ga.zp * (bf ? 2 : 4);
        g.b_t = bf ? kBF16 : kF32; g.sbk = int64_t(H) * ga.zp; g.sbn = 1;
        g.C = wv.dW + int64_t(h) * ga.F * wv.lddw; g.ldc = wv.lddw;
        g.M = ga.F; g.N = ga.cols; g.K = ga.icap; g.K_dev = it.n;
        g.accumulate = 1; g.k_chunk = 256;    // short k-chunks: the loop is latency bound
        if (ga.cols > 0) CK(c, launch_simt_gemm(g, c->stream));
      }
      c->launches++;
    }
    if (ga.cols > 0) {
      launch_pdl(gat_fold_kernel, dim3(L.d_out), dim3(256), 0, c->stream, wv.Wf, wv.ldf,
                 static_cast<const float*>(ga.a_src), static_cast<const float*>(ga.a_dst),
                 static_cast<const float*>(ga.dwt), H, ga.F, ga.cols, wv.dW, wv.lddw, ga.da_src, ga.da_dst);
      CK(c, cudaGetLastError());
      c->launches++;
    }
  }
  return APT_OK;
}

}  // namespace apt
