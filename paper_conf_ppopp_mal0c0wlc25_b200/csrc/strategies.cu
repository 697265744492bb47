// strategies.cu -- the first GNN layer under NFP, SNP and DNP (Fig. 3;
// engine stages Permute / Shuffle / Execute / Reshuffle; Fig. 5 tensor
// partitioning).  GDP is the plain path in trainer.cu.
//
// Every rank is a *requester* (it sampled the layer-1 rows of its own seeds and
// needs their h^1 for the upper layers) and an *owner* (it computes the
// layer-1 work items assigned to it):
//
//   DNP  item (r, i, v) goes to owner part(v): the owner
//        aggregates all sampled sources of v (local rows + NVLink halo) and
//        stores the complete h^1 row (bias, ReLU) into the requester's buffer.
//   SNP  item (r, i, v) goes to every partition c holding >= 1 sampled source of v
//        (P:126): owner c aggregates only its own sources, divided by the
//        full sampled degree (the partial P~_c of §8(a) S7), projects it and adds
//        the partial pre-activation into the requester's buffer; the requester
//        adds the bias and applies the ReLU once, after the sum (reading Z10).
//   NFP  every item goes to every rank (AllBroadcast); rank c aggregates
//        its feature-column slice [lo_c, hi_c) and multiplies it with its
//        column slice of W^1 (column-owned, Fig. 5); partial
//        pre-activations are summed at the requester (reading Z15).
//
// Shuffle (S5) ships (requester, row, node id) triples; the owner re-samples the
// node with the same Philox key, which reproduces the requester's sample bit for
// bit (reading Z2 / Z18), instead of shipping edge lists.  Reshuffle (S9) is the
// routed epilogue of the projection: each output row is stored (DNP) or
// vector-reduced (SNP/NFP) straight into the requester's buffer -- a local
// address in the emulated job, an NVLink peer address in a multi-GPU one.
// Backward (S11): owners gather g = dL/dpre of their items from the requesters,
// compute dW^1 += g^T Z on tcgen05 (or exact fp32), the requester adds db^1;
// dW^1 is all-reduced for DNP/SNP, column-owned (never reduced) for NFP.
#include <algorithm>
#include <type_traits>
#include <vector>

#include "common.cuh"
#include "trainer.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what);
FeatView feat_view(const apt_fstore* f, int r);
}  // namespace apt

#define CK(ctx, expr)                                        \
  do {                                                       \
    apt_status _s = ::apt::check_cuda((ctx), (expr), #expr); \
    if (_s != APT_OK) return _s;                             \
  } while (0)

namespace apt {

static int64_t grid_n(int64_t n, int t = 256) { return grid_cap(ceil_div(n, t), 16); }

struct WorkTab {
  int32_t* const* n;
  int32_t* const* rank;
  int32_t* const* row;
  int32_t* const* gid;
};

// Permute + Shuffle (S4/S5): requester `req` pushes its layer-1 rows to owners.
// mode 0 DNP (owner part(v)), 1 SNP (partitions of the sampled sources), 2 NFP (all).
__global__ void permute_kernel(int mode, int req, int C, const int32_t* __restrict__ dst,
                               const int32_t* __restrict__ n_dst, const int32_t* __restrict__ cnt,
                               const int32_t* __restrict__ nbr, int k, const int32_t* __restrict__ part, WorkTab w) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_dst;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int v = dst[i];
    uint32_t mask;
    if (mode == 0) {
      mask = 1u << part[v];
    } else if (mode == 1) {
      mask = 0;
      const int c = cnt[i];
      for (int e = 0; e < c; ++e) mask |= 1u << part[nbr[i * k + e]];
    } else {
      mask = (1u << C) - 1u;
    }
    while (mask) {
      const int o = __ffs(mask) - 1;
      mask &= mask - 1;
      const int pos = atomicAdd(w.n[o], 1);
      w.rank[o][pos] = req;
      w.row[o][pos] = int32_t(i);
      w.gid[o][pos] = v;
    }
  }
}

// Owner: g rows of its items gathered from the requesters (reverse Shuffle, S11).
// bf16 rows of gb_pitch (16-B vectors), tail of the last 64-row block zeroed.
__global__ void gather_g_bf16_kernel(uint16_t* const* __restrict__ src, int64_t pitch, const int32_t* __restrict__ rank,
                                     const int32_t* __restrict__ row, const int32_t* __restrict__ n_p, int64_t max_n,
                                     uint16_t* __restrict__ out) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int64_t rows = std::min<int64_t>(max_n, round_up(n, 64));
  const int V = int(pitch / 8);
  const int64_t total = rows * V;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = t / V;
    const int j = int(t - i * V);
    uint4 v = make_uint4(0, 0, 0, 0);
    if (i < n) v = *reinterpret_cast<const uint4*>(src[rank[i]] + int64_t(row[i]) * pitch + j * 8);
    *reinterpret_cast<uint4*>(out + i * pitch + j * 8) = v;
  }
}

__global__ void gather_g_f32_kernel(float* const* __restrict__ src, int64_t pitch, const int32_t* __restrict__ rank,
                                    const int32_t* __restrict__ row, const int32_t* __restrict__ n_p,
                                    float* __restrict__ out) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int V = int(pitch / 4);
  const int64_t total = n * V;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = t / V;
    const int j = int(t - i * V);
    *reinterpret_cast<float4*>(out + i * pitch + j * 4) =
        *reinterpret_cast<const float4*>(src[rank[i]] + int64_t(row[i]) * pitch + j * 4);
  }
}

// Requester (SNP / NFP): h = act(sum of partial pre-activations + b), in place (Z10).
__global__ void bias_act_kernel(float* __restrict__ H, int64_t pitch, int dim, const float* __restrict__ b, int relu,
                                const int32_t* __restrict__ n_p) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int64_t total = n * dim;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / dim;
    const int c = int(t - r * dim);
    float v = H[r * pitch + c] + b[c];
    H[r * pitch + c] = relu ? fmaxf(v, 0.f) : v;
  }
}

// db[c] += sum_r g[r][c] over rows r < n (requester-side bias gradient of the
// partial strategies).  Thread = (row lane, 4-column quad); block partials are
// folded in shared memory and added with one atomic per column.
template <typename T>
__global__ void __launch_bounds__(256) colsum_kernel2(const T* __restrict__ g, int64_t pitch, int dim,
                                                      const int32_t* __restrict__ n_p, float* __restrict__ out) {
  APT_PDL_PROLOGUE();
  __shared__ float red[256 * 4];
  const int64_t n = *n_p;
  const int V = int(ceil_div(dim, 4));
  const int rows_per = max(1, 256 / V);
  const int q = threadIdx.x % V, rl = threadIdx.x / V;
  float s[4] = {0.f, 0.f, 0.f, 0.f};
  if (rl < rows_per) {
    for (int64_t r = int64_t(blockIdx.x) * rows_per + rl; r < n; r += int64_t(gridDim.x) * rows_per) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = q * 4 + j;
        if (c < dim) {
          if constexpr (sizeof(T) == 2) s[j] += __uint_as_float(uint32_t(g[r * pitch + c]) << 16);
          else s[j] += float(g[r * pitch + c]);
        }
      }
    }
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) red[threadIdx.x * 4 + j] = s[j];
  __syncthreads();
  if (threadIdx.x < V) {
    for (int j = 0; j < 4; ++j) {
      const int c = threadIdx.x * 4 + j;
      if (c >= dim) break;
      float a = 0.f;
      for (int r = 0; r < rows_per; ++r) a += red[(r * V + threadIdx.x) * 4 + j];
      atomicAdd(out + c, a);
    }
  }
}

apt_status launch_colsum2(apt_ctx* c, const void* g, bool bf16, int64_t pitch, int dim, const int32_t* n_dev,
                                 float* out) {
  if (dim > 1024) {   // column chunks of 1024
    for (int c0 = 0; c0 < dim; c0 += 1024) {
      const void* gc = bf16 ? static_cast<const void*>(static_cast<const uint16_t*>(g) + c0)
                            : static_cast<const void*>(static_cast<const float*>(g) + c0);
      apt_status s = launch_colsum2(c, gc, bf16, pitch, std::min(1024, dim - c0), n_dev, out + c0);
      if (s != APT_OK) return s;
    }
    return APT_OK;
  }
  const int blocks = 296;
  if (bf16) launch_pdl(colsum_kernel2<uint16_t>, dim3(blocks), dim3(256), 0, c->stream, static_cast<const uint16_t*>(g), pitch, dim, n_dev, out);
  else launch_pdl(colsum_kernel2<float>, dim3(blocks), dim3(256), 0, c->stream, static_cast<const float*>(g), pitch, dim, n_dev, out);
  CK(c, cudaGetLastError());
  c->launches++;
  return APT_OK;
}

template <typename T>
static T* upload_tab(apt_trainer* t, const std::vector<T>& v) {
  T* d = t->arena.alloc<T>(int64_t(v.size()), false);
  if (d) cudaMemcpyAsync(d, v.data(), sizeof(T) * v.size(), cudaMemcpyHostToDevice, t->ctx->stream);
  return d;
}

// ------------------------------------------------------------------ allocation
apt_status strategy_alloc(apt_trainer* t, RankState& rs) {
  apt_ctx* c = t->ctx;
  Arena& A = t->arena;
  const int C = t->world;
  const Layer& L = rs.L[0];
  const Hop& hp = rs.hops[t->K - 1];
  Xchg& x = rs.x;
  x.wcap = int64_t(C) * hp.max_dst;       // every requester's rows at most once per owner
  x.n_work = A.alloc<int32_t>(4, true);
  x.work_rank = A.alloc<int32_t>(x.wcap, false);
  x.work_row = A.alloc<int32_t>(x.wcap, false);
  x.work_gid = A.alloc<int32_t>(x.wcap, false);
  x.wcnt = A.alloc<int32_t>(x.wcap, true);
  x.wnbr = A.alloc<int32_t>(x.wcap * hp.k, false);
  if (t->s == APT_NFP) {
    x.col_lo = t->f->col_lo[rs.rank];
    x.col_hi = t->f->col_hi[rs.rank];
  } else {
    x.col_lo = 0;
    x.col_hi = L.d_in;
  }
  x.w_cols = x.col_hi - x.col_lo;
  const bool bf = t->m.dtype == APT_BF16;
  x.wzb_pitch = round_up(x.w_cols + 1, 8);
  x.wzf_pitch = round_up(std::max(x.w_cols, 1), 4);
  if (bf) {
    x.wZb = A.alloc<uint16_t>(x.wcap * x.wzb_pitch, true);
    x.wGb = A.alloc<uint16_t>(x.wcap * L.gb_pitch, true);
  } else {
    x.wZf = A.alloc<float>(x.wcap * x.wzf_pitch, true);
    x.wGf = A.alloc<float>(x.wcap * L.h_pitch, true);
  }
  if (t->s == APT_NFP) {
    x.ws_pitch = round_up(std::max(x.w_cols, 1), 8);
    x.W1s = A.alloc<float>(int64_t(L.d_out) * std::max(x.w_cols, 1), true);
    x.Wb1s = A.alloc<uint16_t>(int64_t(L.d_out) * x.ws_pitch, true);
    x.dW1s = A.alloc<float>(int64_t(L.d_out) * std::max(x.w_cols, 1), true);
  }
  if (!x.work_gid || !x.wnbr || (bf ? !x.wGb : !x.wGf))
    return set_err(c, APT_E_OOM, "strategy_alloc: out of device memory (%lld work items)", (long long)x.wcap);
  return APT_OK;
}

// Pointer tables over all ranks (after every hosted rank is allocated): the
// hosted ranks' own buffers in an emulated job, CUDA-IPC-mapped peer buffers in a
// job of one process per GPU.
apt_status strategy_tables(apt_trainer* t) {
  const int C = t->world;
  std::vector<float*> h1(C), g1(C);
  std::vector<uint16_t*> gb1(C);
  std::vector<int32_t*> wn(C), wr(C), wrow(C), wg(C);
  if (multiprocess(t->ctx)) {
    RankState& rs = t->R[0];
    auto share = [&](auto& tab, auto* mine) -> apt_status {
      if (!mine) return APT_OK;
      std::vector<void*> v(C, nullptr);
      apt_status s = share_ptr(t->ctx, mine, v.data(), &t->peer_opened);
      for (int p = 0; p < C; ++p) tab[p] = static_cast<std::remove_reference_t<decltype(tab[0])>>(v[p]);
      return s;
    };
    apt_status s;
    if ((s = share(h1, rs.L[0].H)) != APT_OK || (s = share(g1, rs.L[0].G)) != APT_OK ||
        (s = share(gb1, rs.L[0].Gb)) != APT_OK || (s = share(wn, rs.x.n_work)) != APT_OK ||
        (s = share(wr, rs.x.work_rank)) != APT_OK || (s = share(wrow, rs.x.work_row)) != APT_OK ||
        (s = share(wg, rs.x.work_gid)) != APT_OK)
      return s;
  } else {
    for (auto& rs : t->R) {
      h1[rs.rank] = rs.L[0].H;
      g1[rs.rank] = rs.L[0].G;
      gb1[rs.rank] = rs.L[0].Gb;
      wn[rs.rank] = rs.x.n_work;
      wr[rs.rank] = rs.x.work_rank;
      wrow[rs.rank] = rs.x.work_row;
      wg[rs.rank] = rs.x.work_gid;
    }
  }
  t->H1_tab = upload_tab(t, h1);
  t->h1_host = h1;
  t->G1_tab = upload_tab(t, g1);
  t->Gb1_tab = upload_tab(t, gb1);
  t->wn_tab = upload_tab(t, wn);
  t->wrank_tab = upload_tab(t, wr);
  t->wrow_tab = upload_tab(t, wrow);
  t->wgid_tab = upload_tab(t, wg);
  if (!t->wgid_tab) return set_err(t->ctx, APT_E_OOM, "strategy_tables: out of device memory");
  return APT_OK;
}

// ------------------------------------------------------------------ forward
// Owner: re-sample the items' nodes -- the same (seed, node, hop, step) key gives the
// requester's sample bit for bit (readings Z2 / Z18).
apt_status resample_items(apt_trainer* t, RankState& rs) {
  apt_ctx* c = t->ctx;
  Xchg& x = rs.x;
  const Hop& hp = rs.hops[t->K - 1];
  SampleArgs sa{t->g->indptr, t->g->indices, x.work_gid, x.n_work, x.wcap, hp.k,
                philox_key(t->m.sample_seed, kDomSample), t->step_dev, t->K - 1, x.wcnt, x.wnbr};
  CK(c, launch_sample(sa, c->stream));
  c->launches++;
  return APT_OK;
}

static apt_status owner_execute(apt_trainer* t, RankState& rs, bool time_it) {
  apt_ctx* c = t->ctx;
  Xchg& x = rs.x;
  Layer& L = rs.L[0];
  const Hop& hp = rs.hops[t->K - 1];
  const bool bf = t->m.dtype == APT_BF16;
  { apt_status s = resample_items(t, rs); if (s != APT_OK) return s; }
  // Execute (S6+S7): fused gather + mean over the items (SNP: own sources only)
  AggArgs a{};
  a.cnt = x.wcnt; a.nbr = x.wnbr; a.k = hp.k;
  a.n_dst = x.n_work; a.max_dst = x.wcap;
  if (t->s == APT_SNP) { a.filt_part = t->g->part; a.keep_part = rs.rank; }
  if (bf) { a.z_bf16 = x.wZb; a.z_bf16_pitch = x.wzb_pitch; }
  else { a.z_f32 = x.wZf; a.z_f32_pitch = x.wzf_pitch; }
  if (time_it) CK(c, tap_event(t, t->ev[6], c->stream));
  CK(c, launch_agg_fstore(a, feat_view(t->f, rs.rank), c->stream));
  if (time_it) CK(c, tap_event(t, t->ev[7], c->stream));
  c->launches++;
  // Projection with the Reshuffle fused into its epilogue (S8+S9): rows routed to the
  // requesters' h^1 buffers; DNP stores act(Y + b), SNP/NFP add partial Y.
  const bool partial = t->s != APT_DNP;
  const int relu = (!partial && t->K > 1) ? 1 : 0;
  const float* bias = partial ? nullptr : L.b;
  const int Kd = x.w_cols;
  if (bf && tc_gemm_supported(L.d_out, std::max(Kd, 1))) {
    const uint16_t* Wb = t->s == APT_NFP ? x.Wb1s : L.Wb;
    const int64_t wp = t->s == APT_NFP ? x.ws_pitch : L.wb_pitch;
    TcGemmArgs g{x.wZb, x.wzb_pitch, Wb, wp, x.wcap, x.n_work, L.d_out, std::max(Kd, 1), bias, relu,
                 nullptr, L.h_pitch, t->H1_tab, x.work_rank, x.work_row, 0, partial ? 1 : 0};
    CK(c, launch_tc_gemm(g, c->stream));
  } else {
    SimtGemmArgs g{};
    if (bf) { g.A = x.wZb; g.a_t = kBF16; g.sam = x.wzb_pitch; }
    else { g.A = x.wZf; g.a_t = kF32; g.sam = x.wzf_pitch; }
    g.sak = 1;
    if (t->s == APT_NFP) {
      if (bf) { g.B = x.Wb1s; g.b_t = kBF16; g.sbn = x.ws_pitch; }
      else { g.B = x.W1s; g.b_t = kF32; g.sbn = std::max(Kd, 1); }
    } else {
      if (bf) { g.B = L.Wb; g.b_t = kBF16; g.sbn = L.wb_pitch; }
      else { g.B = L.W; g.b_t = kF32; g.sbn = L.d_in; }
    }
    g.sbk = 1;
    g.C = nullptr; g.ldc = L.h_pitch; g.bias = bias; g.M_dev = x.n_work; g.M = x.wcap; g.N = L.d_out; g.K = Kd;
    g.relu = relu; g.accumulate = partial ? 1 : 0;
    g.out_base = t->H1_tab; g.out_rank = x.work_rank; g.out_row = x.work_row;
    if (Kd > 0) CK(c, launch_simt_gemm(g, c->stream));
  }
  c->launches++;
  return APT_OK;
}

// Permute + Shuffle (S4/S5) of the layer-1 rows into the owners' work lists (shared
// by the SAGE and the GAT first layer).  zero_h: also clear the requesters' h^1
// (the partial strategies accumulate into it).
apt_status shuffle_items(apt_trainer* t, bool zero_h) {
  apt_ctx* c = t->ctx;
  const int mode = t->s == APT_DNP ? 0 : t->s == APT_SNP ? 1 : 2;
  const bool partial = zero_h;
  WorkTab w{t->wn_tab, t->wrank_tab, t->wrow_tab, t->wgid_tab};
  // Permute + Shuffle: clear owners' lists (and the requesters' partial-sum buffers),
  // then every requester pushes its layer-1 rows
  for (auto& rs : t->R) {
    CK(c, cudaMemsetAsync(rs.x.n_work, 0, sizeof(int32_t), c->stream));
    if (partial) {
      Layer& L = rs.L[0];
      CK(c, cudaMemsetAsync(L.H, 0, sizeof(float) * L.max_rows * L.h_pitch, c->stream));
    }
  }
  { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // lists cleared everywhere
  for (auto& rs : t->R) {
    const Hop& hp = rs.hops[t->K - 1];
    launch_pdl(permute_kernel, dim3(grid_n(hp.max_dst)), dim3(256), 0, c->stream, mode, rs.rank, t->world, hp.dst, hp.n_dst, hp.cnt,
                                                               hp.nbr, hp.k, t->g->part, w);
    CK(c, cudaGetLastError());
    c->launches++;
  }
  return device_barrier(c);   // every list complete
}

apt_status layer1_fwd_strategy(apt_trainer* t) {
  apt_ctx* c = t->ctx;
  const bool partial = t->s != APT_DNP;
  { apt_status s = shuffle_items(t, partial); if (s != APT_OK) return s; }
  // Execute + Reshuffle on every owner
  bool first = true;
  for (auto& rs : t->R) {
    apt_status s = owner_execute(t, rs, first);
    first = false;
    if (s != APT_OK) return s;
  }
  { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // every h^1 row delivered
  // requesters finish the partial sums: bias once, then the activation (Z10)
  if (partial) {
    for (auto& rs : t->R) {
      Layer& L = rs.L[0];
      launch_pdl(bias_act_kernel, dim3(grid_n(L.max_rows * L.d_out)), dim3(256), 0, c->stream, L.H, L.h_pitch, L.d_out, L.b,
                                                                              t->K > 1 ? 1 : 0, L.n_rows);
      CK(c, cudaGetLastError());
      c->launches++;
    }
  }
  return APT_OK;
}

// ------------------------------------------------------------------ backward
apt_status layer1_bwd_strategy(apt_trainer* t) {
  apt_ctx* c = t->ctx;
  const bool bf = t->m.dtype == APT_BF16;
  // requesters: db^1 = sum of their g rows (bias added once at the requester)
  for (auto& rs : t->R) {
    Layer& L = rs.L[0];
    apt_status s = bf ? launch_colsum2(c, L.Gb, true, L.gb_pitch, L.d_out, L.n_rows, L.db)
                      : launch_colsum2(c, L.G, false, L.h_pitch, L.d_out, L.n_rows, L.db);
    if (s != APT_OK) return s;
  }
  { apt_status s = device_barrier(c); if (s != APT_OK) return s; }   // every requester's g ready
  // owners: gather g of their items, dW^1 (+)= g^T Z
  for (auto& rs : t->R) {
    Xchg& x = rs.x;
    Layer& L = rs.L[0];
    float* dW = t->s == APT_NFP ? x.dW1s : L.dW;
    const int64_t ldw = t->s == APT_NFP ? std::max(x.w_cols, 1) : L.d_in;
    if (t->s == APT_NFP) CK(c, cudaMemsetAsync(x.dW1s, 0, sizeof(float) * L.d_out * std::max(x.w_cols, 1), c->stream));
    if (x.w_cols == 0) continue;
    if (bf) {
      launch_pdl(gather_g_bf16_kernel, dim3(grid_n(x.wcap * (L.gb_pitch / 8))), dim3(256), 0, c->stream, 
          t->Gb1_tab, L.gb_pitch, x.work_rank, x.work_row, x.n_work, x.wcap, x.wGb);
      CK(c, cudaGetLastError());
      if (tc_wgrad_supported(L.d_out, x.w_cols)) {
        TcWgradArgs w{x.wGb, L.gb_pitch, x.wZb, x.wzb_pitch, x.n_work, x.wcap, L.d_out, x.w_cols, dW, nullptr, ldw};
        CK(c, launch_tc_wgrad(w, c->stream));
      } else {
        return set_err(c, APT_E_UNSUPPORTED, "layer-1 weight gradient: d_out %d / cols %d outside the tcgen05 path",
                       L.d_out, x.w_cols);
      }
    } else {
      launch_pdl(gather_g_f32_kernel, dim3(grid_n(x.wcap * (L.h_pitch / 4))), dim3(256), 0, c->stream, 
          t->G1_tab, L.h_pitch, x.work_rank, x.work_row, x.n_work, x.wGf);
      CK(c, cudaGetLastError());
      SimtGemmArgs a{};
      a.A = x.wGf; a.a_t = kF32; a.sam = 1; a.sak = L.h_pitch;
      a.B = x.wZf; a.b_t = kF32; a.sbk = x.wzf_pitch; a.sbn = 1;
      a.C = dW; a.ldc = ldw; a.M = L.d_out; a.N = x.w_cols; a.K = x.wcap; a.K_dev = x.n_work;
      a.accumulate = 1; a.k_chunk = 2048;
      CK(c, launch_simt_gemm(a, c->stream));
    }
    c->launches += 2;
  }
  return APT_OK;
}

}  // namespace apt
