// trainer.cu -- the per-mini-batch training step (sampling -> loading ->
// training) under APT's strategies, for every rank hosted by the ctx.
//
// Step phases:
//   A  S1 seeds of the step, S2/S3 K-hop sampling + compaction (all ranks)
//   B  layer-1 forward under the strategy: Permute / Shuffle / Execute /
//      Reshuffle -- strategies.cu for NFP / SNP / DNP
//   C  S10 upper layers (data parallel) + CE loss
//   D  backward of the upper layers, then the layer-1 backward of the strategy (S11)
//   E  gradient all-reduce across ranks (DDP) + SGD
// Every count stays on the device, every grid is sized by an upper bound:
// the step issues no host synchronisation and can be replayed as a CUDA graph.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <functional>
#include <vector>
#include <cstring>

#include "common.cuh"
#include "trainer.h"

using namespace apt;

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what);
FeatView feat_view(const apt_fstore* f, int r);
// strategies.cu
apt_status strategy_alloc(apt_trainer* t, RankState& rs);
apt_status strategy_tables(apt_trainer* t);
apt_status layer1_fwd_strategy(apt_trainer* t);
apt_status layer1_bwd_strategy(apt_trainer* t);
apt_status gat_alloc(apt_trainer* t, RankState& rs);
apt_status gat_tables(apt_trainer* t);
apt_status gat_layer1_fwd(apt_trainer* t, bool time_it);
apt_status gat_layer1_bwd(apt_trainer* t);
apt_status launch_colsum2(apt_ctx* c, const void* g, bool bf16, int64_t pitch, int dim, const int32_t* n_dev,
                          float* out);

// Floats of the flat gradient buffer [dW1 db1 (da_src1 da_dst1 for a GAT layer 1) dW2 db2 ...].
int64_t grad_floats(const apt_trainer* t, const RankState& rs) {
  int64_t P = 0;
  for (auto& L : rs.L) P += int64_t(L.d_out) * L.d_in + L.d_out;
  if (t->gat_heads) P += 2 * int64_t(rs.L[0].d_out);
  return P;
}
// ... of its layer-1 part
static int64_t grad_floats_l1(const apt_trainer* t) {
  const Layer& L = t->R[0].L[0];
  return int64_t(L.d_out) * L.d_in + L.d_out + (t->gat_heads ? 2 * int64_t(L.d_out) : 0);
}
}  // namespace apt

#define CK(ctx, expr)                                        \
  do {                                                       \
    apt_status _s = ::apt::check_cuda((ctx), (expr), #expr); \
    if (_s != APT_OK) return _s;                             \
  } while (0)

namespace apt {

// One process per GPU: out[i] = sum over ranks of tab[r][i] (peer loads over NVLink);
// the caller fences with device barriers before (peers' gradients complete) and
// after (everyone has read them) and copies out -> own buffer.
__global__ void allreduce_gather_kernel(float* const* tab, int C, int64_t n, float* __restrict__ out) {
  APT_PDL_PROLOGUE();
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    float s = 0.f;
    for (int r = 0; r < C; ++r) s += tab[r][i];   // fixed rank order: every rank gets identical sums
    out[i] = s;
  }
}

__global__ void allreduce_sum_kernel(float* const* tab, int C, int64_t n) {
  APT_PDL_PROLOGUE();
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    float s = 0.f;
    for (int r = 0; r < C; ++r) s += tab[r][i];
    for (int r = 0; r < C; ++r) tab[r][i] = s;
  }
}

// Phase events: inside a stream capture they must become external event-record
// nodes (so replays time the phases); outside a capture a plain record.
static cudaError_t record_ev(apt_trainer* t, int i) { return tap_event(t, t->ev[i], t->ctx->stream); }

// The step id enters the device as a kernel argument (no host cell that a later
// call could overwrite before the copy runs); graph replays patch the argument.
__global__ void set_step_kernel(uint64_t* step_dev, uint64_t step) {
  APT_PDL_PROLOGUE(); *step_dev = step; }

// dst[r][0:cols] = src[r][0:cols] for r < *n (device count)
__global__ void copy_rows_kernel(float* __restrict__ dst, int64_t dp, const float* __restrict__ src, int64_t sp, int cols,
                                 const int32_t* __restrict__ n_p) {
  APT_PDL_PROLOGUE();
  const int64_t total = int64_t(*n_p) * cols;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / cols;
    const int c = int(t - r * cols);
    dst[r * dp + c] = src[r * sp + c];
  }
}

// The set_step node of a captured step graph, and its per-replay patch.
static cudaGraphNode_t find_step_node(cudaGraph_t graph) {
  size_t n = 0;
  if (cudaGraphGetNodes(graph, nullptr, &n) != cudaSuccess) return nullptr;
  std::vector<cudaGraphNode_t> nodes(n);
  if (cudaGraphGetNodes(graph, nodes.data(), &n) != cudaSuccess) return nullptr;
  for (auto nd : nodes) {
    cudaGraphNodeType ty;
    if (cudaGraphNodeGetType(nd, &ty) != cudaSuccess || ty != cudaGraphNodeTypeKernel) continue;
    cudaKernelNodeParams kp;
    if (cudaGraphKernelNodeGetParams(nd, &kp) == cudaSuccess && kp.func == (void*)set_step_kernel) return nd;
  }
  return nullptr;
}

static cudaError_t patch_step_node(cudaGraphExec_t exec, cudaGraphNode_t node, uint64_t* step_dev, uint64_t step) {
  void* args[2] = {&step_dev, &step};
  cudaKernelNodeParams kp{};
  kp.func = (void*)set_step_kernel;
  kp.gridDim = dim3(1);
  kp.blockDim = dim3(1);
  kp.kernelParams = args;
  return cudaGraphExecKernelNodeSetParams(exec, node, &kp);
}

__global__ void zero_rows_kernel(float* p, int64_t pitch, const int32_t* n_p) {
  APT_PDL_PROLOGUE();
  const int64_t total = int64_t(*n_p) * pitch;
  float4* q = reinterpret_cast<float4*>(p);
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total / 4; t += int64_t(gridDim.x) * blockDim.x)
    q[t] = make_float4(0.f, 0.f, 0.f, 0.f);
}

static int64_t blocks_for(int64_t n) { return grid_cap(ceil_div(n, 256), 16); }

// Projection dispatch: tcgen05 (bf16 mode) or exact fp32 CUDA cores.
apt_status project(apt_trainer* t, const Layer& L, const void* Zb, const float* Zf, int64_t z_pitch_b,
                   int64_t z_pitch_f, const int32_t* n_rows, int64_t max_rows, int K, const float* W, const uint16_t* Wb,
                   const float* bias, int relu, float* Y, float* const* out_base, const int32_t* out_rank,
                   const int32_t* out_row) {
  apt_ctx* c = t->ctx;
  if (t->m.dtype == APT_BF16 && tc_gemm_supported(L.d_out, K)) {
    TcGemmArgs a{static_cast<const uint16_t*>(Zb), z_pitch_b, Wb, L.wb_pitch, max_rows, n_rows, L.d_out, K,
                 bias, relu, Y, L.h_pitch, out_base, out_rank, out_row, 0};
    if (relu && L.Mk && !out_rank) { a.mask = L.Mk; a.mask_pitch = L.mk_pitch; }   // ReLU bits for the backward
    if (Y == L.H) L.mk_valid = a.mask != nullptr;
    if (Y == L.H && L.Hb && !out_rank) { a.Yb = L.Hb; a.yb_pitch = L.hb_pitch; }   // R11: bf16 only
    a.b_early = 1;   // the step's weights change only in the SGD at its end
    CK(c, launch_tc_gemm(a, c->stream));
  } else {
    if (out_rank) return set_err(c, APT_E_UNSUPPORTED, "routed epilogue needs the tcgen05 path");
    SimtGemmArgs a{};
    if (t->m.dtype == APT_BF16) { a.A = Zb; a.a_t = kBF16; a.sam = z_pitch_b; a.B = Wb; a.b_t = kBF16; a.sbn = L.wb_pitch; }
    else { a.A = Zf; a.a_t = kF32; a.sam = z_pitch_f; a.B = W; a.b_t = kF32; a.sbn = L.d_in; }
    a.sak = 1; a.sbk = 1;
    a.C = Y; a.ldc = L.h_pitch; a.bias = bias; a.M_dev = n_rows; a.M = max_rows; a.N = L.d_out; a.K = K; a.relu = relu;
    CK(c, launch_simt_gemm(a, c->stream));
    if (Y == L.H && L.Hb) {   // R11: the bf16 copy the next layer and the backward read
      CK(c, launch_to_bf16(L.H, L.h_pitch, L.Hb, L.hb_pitch, L.d_out, n_rows, max_rows, c->stream));
      c->launches++;
    }
  }
  c->launches++;
  return APT_OK;
}

// Reading R11: layer-1 producers that write fp32 H (the strategies' Reshuffle, GAT, the
// fused opt-in kernel) hand the next layer its bf16 copy.
apt_status hidden1_to_bf16(apt_trainer* t) {
  apt_ctx* c = t->ctx;
  for (auto& rs : t->R) {
    Layer& L = rs.L[0];
    if (!L.Hb) continue;
    CK(c, launch_to_bf16(L.H, L.h_pitch, L.Hb, L.hb_pitch, L.d_out, L.n_rows, L.max_rows, c->stream));
    c->launches++;
  }
  return APT_OK;
}

// dW (+)= G^T Z over the device-counted rows; db += colsum(G)
apt_status weight_grad(apt_trainer* t, const Layer& L, const float* G, int64_t g_pitch, const void* Z, bool z_bf16,
                       int64_t z_pitch, const int32_t* n_rows, int64_t max_rows, int d_in, float* dW, float* db,
                       int64_t dW_ld, cudaStream_t st = nullptr) {
  apt_ctx* c = t->ctx;
  if (!st) st = c->stream;
  if (z_bf16 && L.Gb && tc_wgrad_supported(L.d_out, d_in)) {
    // tcgen05: dW = Gb^T Zb with db from Z's all-ones column d_in
    TcWgradArgs w{L.Gb, L.gb_pitch, static_cast<const uint16_t*>(Z), z_pitch, n_rows, max_rows, L.d_out, d_in,
                  dW, db};
    CK(c, launch_tc_wgrad(w, st));
    c->launches++;
    return APT_OK;
  }
  // fp32 mode: 3xTF32 tensor cores (gemm_tc_gen.cu), db from Z's all-ones column d_in
  if (!z_bf16 && z_pitch > d_in) {
    SimtGemmArgs a{};
    a.A = G; a.a_t = kF32; a.sam = 1; a.sak = g_pitch;
    a.B = Z; a.b_t = kF32; a.sbk = z_pitch; a.sbn = 1;
    a.C = dW; a.ldc = dW_ld; a.M = L.d_out; a.N = d_in + (db ? 1 : 0); a.K = max_rows; a.K_dev = n_rows;
    a.accumulate = 1;
    if (tc_gen_supported(a)) {
      CK(c, launch_tc_gen_gemm(a, db ? d_in : -1, db, st));
      c->launches++;
      return APT_OK;
    }
  }
  // CUDA cores (dims or strides past the tensor-core kernels): in bf16 mode the hidden
  // layers' gradient exists only as its bf16 copy Gb (the pull kernel writes no fp32 G)
  SimtGemmArgs a{};
  const bool gb = z_bf16 && L.Gb;
  if (gb) { a.A = L.Gb; a.a_t = kBF16; a.sak = L.gb_pitch; }
  else { a.A = G; a.a_t = kF32; a.sak = g_pitch; }
  a.sam = 1;
  a.B = Z; a.b_t = z_bf16 ? kBF16 : kF32; a.sbk = z_pitch; a.sbn = 1;
  a.C = dW; a.ldc = dW_ld; a.M = L.d_out; a.N = d_in; a.K = max_rows; a.K_dev = n_rows;
  a.accumulate = 1; a.k_chunk = 256;      // short k-chunks: the simt k-loop is latency bound
  CK(c, launch_simt_gemm(a, st));
  if (db) {
    if (gb) {
      cudaStream_t keep = c->stream;
      c->stream = st;
      apt_status s2 = launch_colsum2(c, L.Gb, true, L.gb_pitch, L.d_out, n_rows, db);
      c->stream = keep;
      if (s2 != APT_OK) return s2;
    } else {
      CK(c, launch_colsum(G, g_pitch, L.d_out, n_rows, max_rows, db, st));
    }
  }
  c->launches += db ? 2 : 1;
  return APT_OK;
}

}  // namespace apt

extern "C" {

apt_status apt_trainer_destroy(apt_trainer* t);

namespace apt {
// layer_only: a first-layer session of apt_layer_fwd (no labels, no loss)
apt_status trainer_create(apt_ctx* c, const apt_graph* g, const apt_fstore* f, const apt_model_desc* m,
                          apt_strategy s, const int32_t* labels, apt_trainer** out, bool layer_only);
}

apt_status apt_trainer_create(apt_ctx* c, const apt_graph* g, const apt_fstore* f, const apt_model_desc* m,
                              apt_strategy s, const int32_t* labels, apt_trainer** out) {
  if (!labels) return set_err(c, APT_E_INVALID, "apt_trainer_create: labels is null");
  return apt::trainer_create(c, g, f, m, s, labels, out, false);
}

apt_status apt::trainer_create(apt_ctx* c, const apt_graph* g, const apt_fstore* f, const apt_model_desc* m,
                               apt_strategy s, const int32_t* labels, apt_trainer** out, bool layer_only) {
  if (!c || !g || !f || !m || (!labels && !layer_only) || !out || m->n_layers < 1 || m->n_layers > APT_MAX_LAYERS || m->batch < 1 ||
      s < APT_GDP || s > APT_DNP)
    return set_err(c, APT_E_INVALID, "apt_trainer_create: bad arguments");
  if (m->dims[0] != f->dim) return set_err(c, APT_E_INVALID, "apt_trainer_create: dims[0]=%d != store dim %d", m->dims[0], f->dim);
  if (c->world > 1 && s == APT_NFP && f->layout != APT_NFP)
    return set_err(c, APT_E_INVALID, "apt_trainer_create: NFP needs an NFP (column-sharded) store");
  if (c->world > 1 && s != APT_NFP && f->layout == APT_NFP)
    return set_err(c, APT_E_INVALID, "apt_trainer_create: row strategies need a row-sharded store");
  for (int l = 0; l < m->n_layers; ++l)
    if (m->fanouts[l] < 1 || m->fanouts[l] > 256 || m->dims[l + 1] < 1)
      return set_err(c, APT_E_INVALID, "apt_trainer_create: fanout/dim out of range");
  if (m->gat_heads < 0 || m->gat_heads > 8 || (m->gat_heads & (m->gat_heads - 1)) ||
      (m->gat_heads && m->dims[1] % m->gat_heads))
    return set_err(c, APT_E_INVALID, "apt_trainer_create: gat_heads must be 0, 1, 2, 4 or 8 and divide dims[1]");
  auto* t = new apt_trainer();
  t->ctx = c;
  t->gat_heads = m->gat_heads;
  ctx_retain(c);
  t->g = g;
  t->f = f;
  t->m = *m;
  t->s = s;
  t->K = m->n_layers;
  t->world = c->world;
  Arena& A = t->arena;
  const int K = t->K, C = t->world;
  t->labels = labels ? A.alloc<int32_t>(g->n, false) : nullptr;
  t->step_cells = A.alloc<uint64_t>(2, true);   // step id of sample set 0 / 1
  t->step_dev = t->step_cells;
  t->hb_len = 1 + int64_t(C) * m->batch;
  t->hb_dev = A.alloc<int32_t>(2 * t->hb_len, true);
  CK(c, cudaMallocHost(reinterpret_cast<void**>(&t->hb_pinned), sizeof(int32_t) * 2 * t->hb_len));
  CK(c, cudaMallocHost(reinterpret_cast<void**>(&t->loss_pinned), sizeof(float) * 2 * APT_MAX_RANKS));
  for (int q = 0; q < 2; ++q) CK(c, cudaEventCreateWithFlags(&t->ev_done[q], cudaEventDisableTiming));
  if (labels) CK(c, cudaMemcpyAsync(t->labels, labels, sizeof(int32_t) * g->n, cudaMemcpyHostToDevice, c->stream));
  const int64_t n_words = ceil_div(g->n, 32);
  // upper bounds per hop.  SNP/DNP seeds follow the partition: up to C*B on one rank.
  const int64_t B0 = (s == APT_SNP || s == APT_DNP) ? int64_t(C) * m->batch : m->batch;
  t->R.resize(c->n_local);
  for (int li = 0; li < c->n_local; ++li) {
    RankState& rs = t->R[li];
    rs.rank = c->emulated ? li : c->rank;
    rs.loss = A.alloc<float>(4, true);
    rs.ce_ws = A.alloc<int32_t>(kCeMaxBlocks + 4, true);
    rs.dst_bm = A.alloc<uint32_t>(n_words, true);
    rs.new_bm = A.alloc<uint32_t>(n_words, true);
    rs.pos = A.alloc<int32_t>(g->n, false);
    rs.partials = A.alloc<int32_t>(2 * ceil_div(n_words, kScanWsTile) + 8, false);
    for (int q = 0; q < 2; ++q) {
      SampleSet& ss = rs.sset[q];
      ss.seeds = A.alloc<int32_t>(std::max<int64_t>(B0, int64_t(C) * m->batch), false);
      ss.small = A.alloc<int32_t>(16, true);
      ss.step_cell = t->step_cells + q;
      ss.hops.resize(K);
      int64_t maxF = B0;
      const int32_t* dst = ss.seeds;
      const int32_t* n_dst = ss.small;
      for (int h = 0; h < K; ++h) {
        Hop& hp = ss.hops[h];
        hp.k = m->fanouts[K - 1 - h];
        hp.max_dst = maxF;
        hp.max_src = std::max<int64_t>(maxF, std::min<int64_t>(maxF * (1 + hp.k), g->n));
        hp.dst = dst;
        hp.n_dst = n_dst;
        hp.cnt = A.alloc<int32_t>(maxF, true);
        hp.nbr = A.alloc<int32_t>(maxF * hp.k, false);
        hp.counts = A.alloc<int32_t>(4, true);
        hp.part2 = A.alloc<int32_t>(2 * ceil_div(maxF, kScanWsTile) + 8, false);
        if (h + 1 < K) {   // the layer-1 hop is consumed in ELL form (fused gather), no CSR needed
          hp.src = A.alloc<int32_t>(hp.max_src, false);
          hp.indptr = A.alloc<int32_t>(maxF + 1, true);
          hp.indices = A.alloc<int32_t>(maxF * hp.k, false);
          hp.csc_cnt = A.alloc<int32_t>(hp.max_src, true);
          hp.csc_ptr = A.alloc<int32_t>(hp.max_src + 1, true);
          hp.csc_dst = A.alloc<int2>(maxF * hp.k, false);
          hp.csc_ws = A.alloc<int32_t>(2 * ceil_div(hp.max_src, kScanWsTile) + 8, false);
        }
        dst = hp.src;
        n_dst = hp.counts;
        maxF = hp.max_src;
      }
    }
    rs.seeds = rs.sset[0].seeds;
    rs.small = rs.sset[0].small;
    rs.hops = rs.sset[0].hops;
    rs.L.resize(K);
    for (int l = 1; l <= K; ++l) {
      Layer& L = rs.L[l - 1];
      const Hop& hp = rs.hops[K - l];
      L.d_in = m->dims[l - 1];
      L.d_out = m->dims[l];
      L.zf_pitch = round_up(L.d_in + 1, 4);    // + the all-ones bias-gradient column (fp32 mode)
      L.zb_pitch = round_up(L.d_in + 1, 8);   // + the all-ones bias-gradient column
      L.gb_pitch = round_up(L.d_out, 8);
      L.h_pitch = round_up(L.d_out, 4);
      L.wb_pitch = round_up(L.d_in, 8);
      L.max_rows = hp.max_dst;
      L.n_rows = hp.n_dst;
      if (m->dtype == APT_BF16) L.Zb = A.alloc<uint16_t>(L.max_rows * L.zb_pitch, true);
      else L.Zf = A.alloc<float>(L.max_rows * L.zf_pitch, true);
      L.H = A.alloc<float>(L.max_rows * L.h_pitch, true);
      if (m->dtype == APT_BF16 && l < K) {   // reading R11: hidden activations stored in bf16
        L.hb_pitch = round_up(L.d_out, 8);
        L.Hb = A.alloc<uint16_t>(L.max_rows * L.hb_pitch, true);
      }
      L.G = A.alloc<float>(L.max_rows * L.h_pitch, true);
      if (m->dtype == APT_BF16) L.Gb = A.alloc<uint16_t>(L.max_rows * L.gb_pitch, true);
      // ReLU bit masks of the bf16 hidden layers (APT_RELU_BITS=1, opt-in): the direct
      // epilogue writes each row's 64 bits per warp as one 8-byte store, and the mean's
      // backward reads 32 B of bits per row instead of the 512-B bf16 row of H.  (Round 1
      // measured the staged epilogue's 2-byte mask stores: they cost the projection more
      // than the pull saved -- 78 vs 66 us forward, 72 vs 74 us backward.  Round 2, bits from
      // the direct / TMA-store epilogue: layer-1 forward 40.5 -> 45.0 us, backward -1 us,
      // step 0.1500 -> 0.1550 ms: off by default.)
      static const int relu_bits = [] { const char* v = std::getenv("APT_RELU_BITS"); return v ? atoi(v) : 0; }();
      if (m->dtype == APT_BF16 && l < K && relu_bits) {
        L.mk_pitch = round_up(ceil_div(L.d_out, 16), 4);
        L.Mk = A.alloc<uint16_t>(L.max_rows * L.mk_pitch, true);
      }
      if (l > 1) L.dZ = A.alloc<float>(L.max_rows * L.zf_pitch, true);
      if (l > 1 && m->dtype == APT_BF16) {   // reading R13: the mean's backward reads dZ / deg in bf16
        L.dzb_pitch = round_up(L.d_in, 8);
        L.dZb = A.alloc<uint16_t>(L.max_rows * L.dzb_pitch, true);
      }
      L.W = A.alloc<float>(int64_t(L.d_out) * L.d_in, true);
      L.b = A.alloc<float>(L.d_out, true);
      L.Wb = A.alloc<uint16_t>(int64_t(L.d_out) * L.wb_pitch, true);
    }
    // layer-1 Z per sample set (the pipelined sampling branch aggregates the next batch)
    {
      Layer& L1 = rs.L[0];
      rs.sset[0].z1b = L1.Zb;
      rs.sset[0].z1f = L1.Zf;
      if (L1.Zb) rs.sset[1].z1b = A.alloc<uint16_t>(L1.max_rows * L1.zb_pitch, true);
      if (L1.Zf) rs.sset[1].z1f = A.alloc<float>(L1.max_rows * L1.zf_pitch, true);
    }
    // flat gradient buffer [dW1 db1 dW2 db2 ...] so one all-reduce covers the model
    const int64_t P = grad_floats(t, rs);
    float* grads = A.alloc<float>(P, true);
    int64_t off = 0;
    for (auto& L : rs.L) {
      L.dW = grads + off;
      off += int64_t(L.d_out) * L.d_in;
      L.db = grads + off;
      off += L.d_out;
      if (&L == &rs.L[0] && t->gat_heads) {
        rs.ga.da_src = grads + off;
        rs.ga.da_dst = grads + off + L.d_out;
        off += 2 * int64_t(L.d_out);
      }
    }
    if (!rs.seeds || !rs.pos || !grads) {
      apt_trainer_destroy(t);
      return set_err(c, APT_E_OOM, "apt_trainer_create: out of device memory");
    }
    if (C > 1 && s != APT_GDP) {
      apt_status st = strategy_alloc(t, rs);
      if (st != APT_OK) { apt_trainer_destroy(t); return st; }
    }
    if (t->gat_heads) {
      apt_status st = gat_alloc(t, rs);
      if (st != APT_OK) { apt_trainer_destroy(t); return st; }
    }
  }
  if (C > 1 && s != APT_GDP) {
    apt_status st = strategy_tables(t);
    if (st != APT_OK) { apt_trainer_destroy(t); return st; }
  }
  if (t->gat_heads) {
    apt_status st = gat_tables(t);
    if (st != APT_OK) { apt_trainer_destroy(t); return st; }
  }
  if (multiprocess(c)) {
    // every rank reads every peer's flat gradient buffer in the all-reduce
    std::vector<void*> v(C, nullptr);
    apt_status st = share_ptr(c, t->R[0].L[0].dW, v.data(), &t->peer_opened);
    if (st != APT_OK) { apt_trainer_destroy(t); return st; }
    const int64_t P = grad_floats(t, t->R[0]);
    t->ar_scratch = A.alloc<float>(P, false);
    t->dW_tab = A.alloc<float*>(C, false);
    CK(c, cudaMemcpyAsync(t->dW_tab, v.data(), sizeof(float*) * C, cudaMemcpyHostToDevice, c->stream));
  } else {
    std::vector<float*> tab(C, nullptr);
    for (auto& rs : t->R) tab[rs.rank] = rs.L[0].dW;
    t->dW_tab = A.alloc<float*>(C, false);
    CK(c, cudaMemcpyAsync(t->dW_tab, tab.data(), sizeof(float*) * C, cudaMemcpyHostToDevice, c->stream));
  }
  for (int i = 0; i < 8; ++i) cudaEventCreate(&t->ev[i]);
  {
    // opt-in (A/B): the next batch's layer-1 gather+mean on the sampling branch.
    // Step 0.187 -> 0.179 ms, but the gather then runs beside the latency-bound backward
    // (pull / wgrad: 60 -> 92 us) and its own in-step time rises 30 -> 43 us
    const char* zp = std::getenv("APT_Z_PREFETCH");
    t->z_prefetch = (zp && atoi(zp) != 0) && !t->gat_heads && (C == 1 || s == APT_GDP);
    t->z_where = zp ? std::max(1, atoi(zp)) : 1;
    CK(c, cudaEventCreateWithFlags(&t->ev_zt, cudaEventDisableTiming));
    CK(c, cudaEventCreateWithFlags(&t->ev_zf, cudaEventDisableTiming));
  }
  CK(c, cudaStreamSynchronize(c->stream));
  *out = t;
  return APT_OK;
}

apt_status apt_trainer_destroy(apt_trainer* t) {
  if (!t) return APT_OK;
  cudaStreamSynchronize(t->ctx->stream);
  if (t->gexec) cudaGraphExecDestroy(t->gexec);
  if (t->graph) cudaGraphDestroy(t->graph);
  for (int p = 0; p < 2; ++p)
    for (int u = 0; u < 2; ++u) {
      if (t->gexec_p[p][u]) cudaGraphExecDestroy(t->gexec_p[p][u]);
      if (t->graph_p[p][u]) cudaGraphDestroy(t->graph_p[p][u]);
      if (t->gexec_hp[p][u]) cudaGraphExecDestroy(t->gexec_hp[p][u]);
      if (t->graph_hp[p][u]) cudaGraphDestroy(t->graph_hp[p][u]);
    }
  if (t->gexec_host) cudaGraphExecDestroy(t->gexec_host);
  if (t->graph_host) cudaGraphDestroy(t->graph_host);
  if (t->hb_pinned) cudaFreeHost(t->hb_pinned);
  if (t->loss_pinned) cudaFreeHost(t->loss_pinned);
  if (t->ev_zt) cudaEventDestroy(t->ev_zt);
  if (t->ev_zf) cudaEventDestroy(t->ev_zf);
  for (int q = 0; q < 2; ++q)
    if (t->ev_done[q]) cudaEventDestroy(t->ev_done[q]);
  for (int i = 0; i < 8; ++i)
    if (t->ev[i]) cudaEventDestroy(t->ev[i]);
  apt_ctx* c = t->ctx;
  delete t;
  ctx_release(c);
  return APT_OK;
}

apt_status apt_trainer_set_params(apt_trainer* t, int layer, const float* W, const float* b) {
  if (!t || layer < 1 || layer > t->K || !W || !b) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "set_params: bad args");
  apt_ctx* c = t->ctx;
  for (auto& rs : t->R) {
    Layer& L = rs.L[layer - 1];
    CK(c, cudaMemcpyAsync(L.W, W, sizeof(float) * L.d_out * L.d_in, cudaMemcpyDefault, c->stream));   // host or device
    CK(c, cudaMemcpyAsync(L.b, b, sizeof(float) * L.d_out, cudaMemcpyDefault, c->stream));
    CK(c, launch_to_bf16(L.W, L.d_in, L.Wb, L.wb_pitch, L.d_in, nullptr, L.d_out, c->stream));
    c->launches++;
    if (layer == 1 && rs.x.W1s) {   // NFP: the rank's column slice of W^1 (column-owned)
      const int w = rs.x.w_cols;
      if (w > 0) {
        CK(c, cudaMemcpy2DAsync(rs.x.W1s, sizeof(float) * w, W + rs.x.col_lo, sizeof(float) * L.d_in, sizeof(float) * w,
                                L.d_out, cudaMemcpyDefault, c->stream));
        CK(c, launch_to_bf16(rs.x.W1s, w, rs.x.Wb1s, rs.x.ws_pitch, w, nullptr, L.d_out, c->stream));
        c->launches++;
      }
    }
  }
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

apt_status apt_trainer_get_params(apt_trainer* t, int rank, int layer, float* W, float* b) {
  if (!t || layer < 1 || layer > t->K) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "get_params: bad args");
  for (auto& rs : t->R)
    if (rs.rank == rank) {
      Layer& L = rs.L[layer - 1];
      CK(t->ctx, cudaStreamSynchronize(t->ctx->stream));
      if (W) CK(t->ctx, cudaMemcpy(W, L.W, sizeof(float) * L.d_out * L.d_in, cudaMemcpyDeviceToHost));
      if (W && layer == 1 && rs.x.W1s) {   // NFP: W^1 is column-owned; assemble the hosted slices
        for (auto& o : t->R) {
          if (o.x.w_cols <= 0) continue;
          CK(t->ctx, cudaMemcpy2D(W + o.x.col_lo, sizeof(float) * L.d_in, o.x.W1s, sizeof(float) * o.x.w_cols,
                                  sizeof(float) * o.x.w_cols, L.d_out, cudaMemcpyDeviceToHost));
        }
      }
      if (b) CK(t->ctx, cudaMemcpy(b, L.b, sizeof(float) * L.d_out, cudaMemcpyDeviceToHost));
      return APT_OK;
    }
  return set_err(t->ctx, APT_E_INVALID, "get_params: rank %d not hosted", rank);
}

apt_status apt_trainer_set_attention(apt_trainer* t, const float* a_src, const float* a_dst) {
  if (!t || !a_src || !a_dst) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "set_attention: bad args");
  if (!t->gat_heads) return set_err(t->ctx, APT_E_STATE, "set_attention: layer 1 is not a GAT layer");
  apt_ctx* c = t->ctx;
  for (auto& rs : t->R) {
    CK(c, cudaMemcpyAsync(rs.ga.a_src, a_src, sizeof(float) * rs.L[0].d_out, cudaMemcpyHostToDevice, c->stream));
    CK(c, cudaMemcpyAsync(rs.ga.a_dst, a_dst, sizeof(float) * rs.L[0].d_out, cudaMemcpyHostToDevice, c->stream));
  }
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

apt_status apt_trainer_get_attention(apt_trainer* t, int rank, float* a_src, float* a_dst) {
  if (!t || !a_src || !a_dst) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "get_attention: bad args");
  if (!t->gat_heads) return set_err(t->ctx, APT_E_STATE, "get_attention: layer 1 is not a GAT layer");
  for (auto& rs : t->R)
    if (rs.rank == rank) {
      CK(t->ctx, cudaStreamSynchronize(t->ctx->stream));
      CK(t->ctx, cudaMemcpy(a_src, rs.ga.a_src, sizeof(float) * rs.L[0].d_out, cudaMemcpyDeviceToHost));
      CK(t->ctx, cudaMemcpy(a_dst, rs.ga.a_dst, sizeof(float) * rs.L[0].d_out, cudaMemcpyDeviceToHost));
      return APT_OK;
    }
  return set_err(t->ctx, APT_E_INVALID, "get_attention: rank %d not hosted", rank);
}

apt_status apt_trainer_set_epoch(apt_trainer* t, const int64_t* train, int64_t n_train, uint64_t epoch) {
  if (!t || !train || n_train < 1) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "set_epoch: bad args");
  apt_ctx* c = t->ctx;
  std::vector<int32_t> h(n_train);
  for (int64_t i = 0; i < n_train; ++i) {
    if (train[i] < 0 || train[i] >= t->g->n || (i && train[i] <= train[i - 1]))
      return set_err(c, APT_E_INVALID, "set_epoch: train ids must be ascending and in range");
    h[i] = int32_t(train[i]);
  }
  if (!t->perm || n_train > t->n_train) t->perm = t->arena.alloc<int32_t>(n_train, false);
  t->n_train = n_train;
  t->steps_per_epoch = ceil_div(n_train, int64_t(t->world) * t->m.batch);
  t->primed = -1;   // a prefetched batch belongs to the previous permutation
  t->host_primed = false;
  uint64_t* keys = nullptr;
  void* scratch = nullptr;
  CK(c, cudaMallocAsync(&keys, sizeof(uint64_t) * n_train, c->stream));
  CK(c, cudaMallocAsync(&scratch, radix_sort_pairs_scratch(n_train), c->stream));
  CK(c, cudaMemcpyAsync(t->perm, h.data(), sizeof(int32_t) * n_train, cudaMemcpyHostToDevice, c->stream));
  CK(c, launch_perm_keys(t->perm, n_train, t->m.sample_seed, epoch, keys, c->stream));
  // stable LSD radix sort by key (sort.cu): ties keep the ascending id order (reading O1)
  CK(c, launch_radix_sort_pairs(keys, t->perm, n_train, scratch, c->stream));
  c->launches += 1 + 24;
  CK(c, cudaFreeAsync(keys, c->stream));
  CK(c, cudaFreeAsync(scratch, c->stream));
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

int64_t apt_trainer_steps_per_epoch(const apt_trainer* t) { return t ? t->steps_per_epoch : 0; }

}  // extern "C"

namespace apt {

// Phase A for one rank: seeds + sampling (+ compaction for every hop but the layer-1
// one) into sample set `ss`, on stream `st`.  fork_csc: the block transposes run on the
// side branch (joined before the backward through ev_csc) instead of on `st`.
apt_status phase_sample(apt_trainer* t, RankState& rs, SampleSet& ss, bool from_host_batch, cudaStream_t st,
                        bool fork_csc) {
  apt_ctx* c = t->ctx;
  // background sampling (the next step, pipelined) is confined to a few blocks per SM so
  // that it fills gaps instead of competing with the step's chain for every SM
  static const int64_t bg_cap = [] {
    const char* v = std::getenv("APT_BG_BLOCKS_PER_SM");
    return int64_t(num_sms()) * (v ? std::max(1, atoi(v)) : 8);   // 4 -> 8 with the fused output layer (A/B)
  }();
  const int64_t cap = st == c->samp ? bg_cap : 0;
  {
    // seeds of the step: from the epoch permutation, or from the global batch the host
    // copied in (hb_dev = [n, ids...]); chunk r for GDP/NFP, partition r for SNP/DNP
    const bool by_part = (t->s == APT_SNP || t->s == APT_DNP) && t->world > 1;
    const int32_t* hb = t->hb_dev + (&ss == &rs.sset[1] ? t->hb_len : 0);   // this set's host-batch staging
    SeedArgs sa{from_host_batch ? hb + 1 : t->perm, t->n_train, ss.step_cell, t->steps_per_epoch, t->world,
                rs.rank, t->m.batch, by_part ? 1 : 0, t->g->part, ss.seeds, ss.small, ss.small + 1,
                from_host_batch ? hb : nullptr};
    CK(c, launch_select_seeds(sa, st));
    c->launches++;
  }
  const int64_t n_words = ceil_div(t->g->n, 32);
  for (int h = 0; h < t->K; ++h) {
    Hop& hp = ss.hops[h];
    SampleArgs sa{t->g->indptr, t->g->indices, hp.dst, hp.n_dst, hp.max_dst, hp.k,
                  philox_key(t->m.sample_seed, kDomSample), ss.step_cell, h, hp.cnt, hp.nbr, cap};
    CK(c, launch_sample(sa, st));
    c->launches++;
    if (h + 1 < t->K) {
      CompactArgs ca{hp.dst, hp.n_dst, hp.max_dst, hp.cnt, hp.nbr, hp.k, rs.dst_bm, rs.new_bm, n_words, rs.pos, hp.src,
                     hp.counts, hp.indptr, hp.indices, hp.counts + 1, rs.partials, hp.part2, cap};
      static const int count_in_map = [] { const char* v = std::getenv("APT_CSC_COUNT_IN_MAP"); return v ? atoi(v) : 1; }();
      if (count_in_map) {   // the transpose's in-degrees counted while the indices are mapped
        const int nb = scan_tiles(hp.max_src);
        ca.csc_cnt = hp.csc_cnt; ca.csc_st = reinterpret_cast<uint64_t*>(hp.csc_ws); ca.csc_nb = nb;
        ca.csc_ticket = hp.csc_ws + 2 * nb + 2;
      }
      CK(c, launch_compact(ca, st));
      c->launches += 3;
      // transpose of this block for the pull-form mean backward
      cudaStream_t cs_st = st;
      // the background (next-step) sampling: the transposes on a second low-priority stream,
      // so the next hop's sampling does not wait for them (joined at the branch's end)
      static const int bg_fork = [] { const char* v = std::getenv("APT_BG_CSC_FORK"); return v ? atoi(v) : 1; }();
      if (!fork_csc && bg_fork && st == c->samp) {
        CK(c, cudaEventRecord(c->ev_sfork, st));
        CK(c, cudaStreamWaitEvent(c->samp2, c->ev_sfork, 0));
        cs_st = c->samp2;
        t->bg_csc_forked = true;
      }
      if (fork_csc) {
        CK(c, cudaEventRecord(c->ev_fork, st));
        CK(c, cudaStreamWaitEvent(c->side, c->ev_fork, 0));
        cs_st = c->side;
      }
      CscArgs cs{hp.indptr, hp.indices, hp.n_dst, hp.max_dst, hp.counts + 1, hp.max_dst * hp.k, hp.counts,
                 hp.max_src, hp.csc_cnt, hp.csc_ptr, hp.counts + 2, hp.csc_dst, hp.csc_ws, cap, hp.k,
                 ca.csc_cnt ? 1 : 0};
      CK(c, launch_csc_build(cs, cs_st));
      c->launches += ca.csc_cnt ? 2 : 3;   // (count + scan reset,) scan, fill
    }
  }
  if (fork_csc && t->K > 1) {
    CK(c, cudaEventRecord(c->ev_csc, c->side));
    t->csc_forked = true;
  }
  return APT_OK;
}

apt_status sample_all(apt_trainer* t, int q, bool host_batch, cudaStream_t st, bool fork_csc) {
  for (auto& rs : t->R) {
    apt_status s = phase_sample(t, rs, rs.sset[q], host_batch, st, fork_csc);
    if (s != APT_OK) return s;
  }
  return APT_OK;
}

// Make sample set q the one the compute phases read (host-side pointer switch; a
// captured graph keeps the pointers of its parity).
void activate(apt_trainer* t, int q) {
  for (auto& rs : t->R) {
    SampleSet& ss = rs.sset[q];
    rs.seeds = ss.seeds;
    rs.small = ss.small;
    rs.hops = ss.hops;
    for (int l = 1; l <= t->K; ++l) rs.L[l - 1].n_rows = ss.hops[t->K - l].n_dst;
    if (ss.z1b) rs.L[0].Zb = ss.z1b;
    if (ss.z1f) rs.L[0].Zf = ss.z1f;
  }
  t->step_dev = t->step_cells + q;
  t->parity = q;
}

// Where the next step's sampling branch forks off the step (A/B): 0 at the
// step's start (default), 1 after the layer-1 forward (the gather+aggregate then runs
// alone: 34.6 -> 33.4 us, but the sampling lands on the critical path: step 0.231 -> 0.241 ms),
// 2 after the layer-1 gather (before its projection).
static int sample_fork_point() {
  static const int v = [] { const char* e = std::getenv("APT_SAMPLE_FORK"); return e ? atoi(e) : 0; }();
  return v;
}

// The layer-1 gather+mean of sample set q of one rank (local + peer rows) into the
// set's Z, on stream st; time_it: bracketed by the phase events 6 / 7 (on st).
apt_status agg_l1_set(apt_trainer* t, RankState& rs, int q, cudaStream_t st, bool time_it) {
  apt_ctx* c = t->ctx;
  const Layer& L = rs.L[0];
  const SampleSet& ss = rs.sset[q];
  const Hop& hp = ss.hops[t->K - 1];
  const FeatView fv = feat_view(t->f, rs.rank);
  AggArgs a{};
  a.cnt = hp.cnt; a.nbr = hp.nbr; a.k = hp.k;
  a.n_dst = hp.n_dst; a.max_dst = hp.max_dst; a.dim = L.d_in;
  if (t->m.dtype == APT_BF16) { a.z_bf16 = ss.z1b; a.z_bf16_pitch = L.zb_pitch; a.z_ones = 1; }
  else { a.z_f32 = ss.z1f; a.z_f32_pitch = L.zf_pitch; a.z_ones = 1; }
  // beside the step (the sampling branch): a capped grid leaves registers for the chain
  static const int zbg = [] { const char* v = std::getenv("APT_ZBG_BPSM"); return v ? atoi(v) : 0; }();
  if (st == c->samp) a.bpsm = zbg;
  // the dominant kernel's own events: on the tap branch (default) or in the chain on the
  // launching stream (APT_AGG_EV_CHAIN=1: exact bracket, but no PDL edge into the projection)
  static const int agg_chain = [] { const char* v = std::getenv("APT_AGG_EV_CHAIN"); return v ? atoi(v) : 0; }();
  auto rec = [&](int i) { return tap_event(t, t->ev[i], st, agg_chain != 0); };
  if (time_it) CK(c, rec(6));
  CK(c, launch_agg_fstore(a, fv, st));
  c->launches++;
  if (time_it) CK(c, rec(7));
  return APT_OK;
}

// The layer-1 aggregation of the batch in set q for every hosted rank on stream st
// (the pipelined sampling branch: it depends only on the batch and the static store).
apt_status prefetch_z(apt_trainer* t, int q, cudaStream_t st) {
  bool first = true;
  for (auto& rs : t->R) {
    apt_status s = agg_l1_set(t, rs, q, st, first);
    first = false;
    if (s != APT_OK) return s;
  }
  return APT_OK;
}

// GDP layer-1 forward on one rank: the fused gather+mean (local + peer rows) -- unless
// the pipelined sampling branch already aggregated this batch (z_ready) -- then the
// projection.
apt_status layer1_fwd_gdp(apt_trainer* t, RankState& rs, bool time_it) {
  Layer& L = rs.L[0];
  if (!t->z_ready) {
    apt_status s = agg_l1_set(t, rs, t->parity, t->ctx->stream, time_it);
    if (s != APT_OK) return s;
  }
  if (t->deferred_fork && sample_fork_point() >= 2 && &rs == &t->R.back()) {
    // the next step's sampling forks after the layer-1 gather (the gather runs alone)
    std::function<apt_status()> f = std::move(t->deferred_fork);
    t->deferred_fork = nullptr;
    apt_status s = f();
    if (s != APT_OK) return s;
  }
  return project(t, L, L.Zb, L.Zf, L.zb_pitch, L.zf_pitch, L.n_rows, L.max_rows, L.d_in, L.W, L.Wb, L.b,
                 t->K > 1 ? 1 : 0, L.H, nullptr, nullptr, nullptr);
}

// Reading R13 (bf16 mode): the projection's backward writes dZ / deg as bf16 rows for
// the mean's backward.  APT_BF16_DZ=0 keeps fp32 rows (A/B).
static bool bf16_dz_enabled() {
  const char* e = std::getenv("APT_BF16_DZ");
  return !e || atoi(e) != 0;
}

// Upper layers l = 2..K (data parallel) + CE loss on one rank.
apt_status upper_fwd_loss(apt_trainer* t, RankState& rs) {
  apt_ctx* c = t->ctx;
  t->out_dz_fused = false;
  for (int l = 2; l <= t->K; ++l) {
    Layer& L = rs.L[l - 1];
    const Layer& P = rs.L[l - 2];
    const Hop& hp = rs.hops[t->K - l];
    if (l == t->K && t->m.dtype == APT_BF16 && P.Hb && L.Zb && !L.Hb && L.Gb &&
        out_fused_supported(L.d_in, L.d_out, L.max_rows)) {
      // the output layer's mean, projection and loss in one kernel (outfused.cu)
      OutFusedArgs o{hp.indptr, hp.indices, P.Hb, P.hb_pitch, hp.n_dst, hp.max_dst, L.d_in, L.d_out,
                     L.Zb, L.zb_pitch, L.Wb, L.wb_pitch, L.b, L.H, L.h_pitch,
                     rs.seeds, t->labels, rs.small + 1, rs.loss, L.G, L.h_pitch, L.Gb, L.gb_pitch,
                     rs.L[0].dW, grad_floats(t, rs), reinterpret_cast<float*>(rs.ce_ws + 1), rs.ce_ws};
      // dZ^K = (G W) / deg from the same kernel (APT_OUT_DZ=0: the tcgen05 dZ launch, A/B)
      static const int out_dz = [] { const char* v = std::getenv("APT_OUT_DZ"); return v ? atoi(v) : 1; }();
      t->out_dz_fused = out_dz && L.dZb && bf16_dz_enabled() && tc_gemm_supported(L.d_in, L.d_out);
      if (t->out_dz_fused) { o.dzb = L.dZb; o.dzb_pitch = L.dzb_pitch; }
      CK(c, launch_out_fused(o, c->stream));
      c->launches++;
      return APT_OK;
    }
    AggArgs a{};
    a.indptr = hp.indptr; a.indices = hp.indices; a.x = P.H; a.x_pitch = P.h_pitch;
    if (P.Hb) { a.x = nullptr; a.xb = P.Hb; a.x_pitch = P.hb_pitch; }   // R11
    a.n_dst = hp.n_dst; a.max_dst = hp.max_dst; a.dim = L.d_in;
    if (t->m.dtype == APT_BF16) { a.z_bf16 = L.Zb; a.z_bf16_pitch = L.zb_pitch; a.z_ones = 1; }
    // fp32 Z is kept in both modes for the upper layers' weight gradient in fp32 mode
    if (t->m.dtype != APT_BF16) { a.z_f32 = L.Zf; a.z_f32_pitch = L.zf_pitch; a.z_ones = 1; }
    CK(c, launch_agg_csr(a, c->stream));
    c->launches++;
    apt_status s = project(t, L, L.Zb, L.Zf, L.zb_pitch, L.zf_pitch, L.n_rows, L.max_rows, L.d_in, L.W, L.Wb, L.b,
                           l < t->K ? 1 : 0, L.H, nullptr, nullptr, nullptr);
    if (s != APT_OK) return s;
  }
  Layer& LK = rs.L[t->K - 1];
  // the loss kernel also zeroes this rank's gradient accumulators [dW1 db1 dW2 ...]
  // (no memset node between the forward and the backward)
  CK(c, launch_ce_loss(LK.H, LK.h_pitch, LK.d_out, rs.seeds, rs.small, LK.max_rows, t->labels, rs.small + 1, rs.loss,
                       LK.G, LK.h_pitch, LK.Gb, LK.gb_pitch, rs.L[0].dW, grad_floats(t, rs), rs.ce_ws, c->stream));
  c->launches++;
  return APT_OK;
}

// Where the upper layers' weight gradients fork off the main chain (APT_WG_FORK; A/B).
static int wg_fork_mode() {
  // A/B with the fused output layer and the background transposes off the sampling chain
  // (0 / 1 / 2): 0.1500 / 0.1514 / 0.1571 ms; before them mode 2 won
  static const int m = [] { const char* e = std::getenv("APT_WG_FORK"); return e ? atoi(e) : 0; }();
  return m;
}

// Backward of layers K..2 on one rank (layer 1's weight gradient is strategy specific).
apt_status upper_bwd(apt_trainer* t, RankState& rs) {
  apt_ctx* c = t->ctx;
  const bool bf = t->m.dtype == APT_BF16;
  std::vector<std::function<apt_status()>> late;
  for (int l = t->K; l >= 2; --l) {
    Layer& L = rs.L[l - 1];
    Layer& P = rs.L[l - 2];
    const Hop& hp = rs.hops[t->K - l];
    // dW_l = G_l^T Z_l is independent of the input-gradient chain: fork it onto the
    // side stream (a parallel branch of the step's graph), joined before the all-reduce.
    // Where the fork sits decides which main-chain kernels it shares the SMs with
    // (wg_fork_mode(): 0 before this layer's dZ, 1 after it, 2 after the last dZ).
    auto fork_wgrad = [t, c, bf, Lp = &L]() -> apt_status {
      const Layer& W = *Lp;
      CK(c, cudaEventRecord(c->ev_fork, c->stream));
      CK(c, cudaStreamWaitEvent(c->side, c->ev_fork, 0));
      return weight_grad(t, W, W.G, W.h_pitch, bf ? static_cast<const void*>(W.Zb) : W.Zf, bf,
                         bf ? W.zb_pitch : W.zf_pitch, W.n_rows, W.max_rows, W.d_in, W.dW, W.db, W.d_in, c->side);
    };
    apt_status s = APT_OK;
    if (wg_fork_mode() == 0 && (s = fork_wgrad()) != APT_OK) return s;
    else if (wg_fork_mode() == 2) late.push_back(fork_wgrad);
    int dz_scaled = 0;
    const uint16_t* dzb = nullptr;
    // dZ = G W  (bf16 mode: tcgen05 with the bf16 weights of the forward, W read N-major as stored)
    if (l == t->K && t->out_dz_fused) {   // already written by the fused output-layer kernel
      dz_scaled = 1;
      dzb = L.dZb;
    } else if (bf && tc_gemm_supported(L.d_in, L.d_out)) {
      TcGemmArgs g{L.Gb, L.gb_pitch, L.Wb, L.wb_pitch, L.max_rows, L.n_rows, L.d_in, L.d_out, nullptr, 0,
                   L.dZ, L.zf_pitch, nullptr, nullptr, nullptr, 1};
      g.row_div_indptr = hp.indptr;   // dZ / deg once per row (the pull then only sums)
      g.b_early = 1;
      if (L.dZb && bf16_dz_enabled()) { g.Yb = L.dZb; g.yb_pitch = L.dzb_pitch; dzb = L.dZb; }   // R13
      CK(c, launch_tc_gemm(g, c->stream));
      dz_scaled = 1;
    } else {
      SimtGemmArgs a{};
      if (bf) { a.A = L.Gb; a.a_t = kBF16; a.sam = L.gb_pitch; }   // bf16 mode: only Gb exists
      else { a.A = L.G; a.a_t = kF32; a.sam = L.h_pitch; }
      a.sak = 1;
      if (bf) { a.B = L.Wb; a.b_t = kBF16; a.sbk = L.wb_pitch; }
      else { a.B = L.W; a.b_t = kF32; a.sbk = L.d_in; }
      a.sbn = 1;
      a.C = L.dZ; a.ldc = L.zf_pitch; a.M_dev = L.n_rows; a.M = L.max_rows; a.N = L.d_in; a.K = L.d_out;
      CK(c, launch_simt_gemm(a, c->stream));
    }
    if (wg_fork_mode() == 1 && (s = fork_wgrad()) != APT_OK) return s;
    if (l == 2) {   // mode 2: every upper layer's weight gradient beside the last mean backward
      for (auto& f : late)
        if ((s = f()) != APT_OK) return s;
    }
    // dH_{l-1}: every source row of the layer-l block pulls its in-edges' dZ / deg
    // (transpose built on the side branch), through the ReLU, straight to G (fp32 mode)
    // or its bf16 copy (bf16 mode)
    if (l == t->K && t->csc_forked) CK(c, cudaStreamWaitEvent(c->stream, c->ev_csc, 0));
    // ReLU bits of H_{l-1} exist when its projection ran on this rank's tcgen05 path
    const bool l1_local = l - 1 > 1 || t->world == 1 || t->s == APT_GDP;
    const uint16_t* mk = (bf && P.Mk && P.mk_valid && l1_local && tc_gemm_supported(P.d_out, P.d_in)) ? P.Mk : nullptr;
    PullArgs pa{hp.csc_ptr, hp.csc_dst, hp.indptr, L.dZ, L.zf_pitch, P.H, P.h_pitch, mk, P.mk_pitch,
                bf ? nullptr : P.G, P.h_pitch, bf ? P.Gb : nullptr, P.gb_pitch, hp.counts, P.max_rows, L.d_in,
                dz_scaled};
    // R11: the mask from bf16 H (bf16 mode always passes H; the pull takes the bits instead
    // where it can, else H)
    if (P.Hb) { pa.h = nullptr; pa.hb = P.Hb; pa.hb_pitch = P.hb_pitch; }
    if (dzb) { pa.dzb = dzb; pa.dzb_pitch = L.dzb_pitch; }                            // R13: bf16 dZ / deg
    CK(c, launch_pull_bwd(pa, c->stream));
    c->launches += 2;
  }
  return APT_OK;
}

apt_status layer1_bwd_gdp(apt_trainer* t, RankState& rs) {
  Layer& L = rs.L[0];
  const bool bf = t->m.dtype == APT_BF16;
  return weight_grad(t, L, L.G, L.h_pitch, bf ? static_cast<const void*>(L.Zb) : L.Zf, bf,
                     bf ? L.zb_pitch : L.zf_pitch, L.n_rows, L.max_rows, L.d_in, L.dW, L.db, L.d_in);
}

// Gradient all-reduce over the ranks (DDP) of the first P floats of the
// flat gradient buffer [dW1 db1 dW2 ...].
apt_status allreduce_grads(apt_trainer* t, int64_t P) {
  apt_ctx* c = t->ctx;
  if (c->emulated) {
    launch_pdl(allreduce_sum_kernel, dim3(blocks_for(P)), dim3(256), 0, c->stream, t->dW_tab, t->world, P);
    CK(c, cudaGetLastError());
    c->launches++;
    return APT_OK;
  }
  apt_status s = device_barrier(c);
  if (s != APT_OK) return s;
  launch_pdl(allreduce_gather_kernel, dim3(blocks_for(P)), dim3(256), 0, c->stream, t->dW_tab, t->world, P, t->ar_scratch);
  CK(c, cudaGetLastError());
  if ((s = device_barrier(c)) != APT_OK) return s;
  CK(c, cudaMemcpyAsync(t->R[0].L[0].dW, t->ar_scratch, sizeof(float) * P, cudaMemcpyDeviceToDevice, c->stream));
  c->launches++;
  return APT_OK;
}

apt_status allreduce_sgd(apt_trainer* t, int update) {
  apt_ctx* c = t->ctx;
  const int64_t P = grad_floats(t, t->R[0]);
  if (t->world > 1) {
    apt_status s = allreduce_grads(t, P);
    if (s != APT_OK) return s;
  }
  if (!update) return APT_OK;
  // one launch per 16 parameter tensors (all layers, all hosted ranks)
  SgdBatch bt{};
  auto add = [&](float* W, const float* dW, int64_t n, uint16_t* Wb, int cols, int64_t bp) -> apt_status {
    bt.seg[bt.n++] = SgdSeg{W, dW, n, Wb, cols, bp};
    if (bt.n == 16) {
      CK(c, launch_sgd_multi(bt, t->m.lr, c->stream));
      c->launches++;
      bt.n = 0;
    }
    return APT_OK;
  };
  for (auto& rs : t->R) {
    for (auto& L : rs.L) {
      apt_status st;
      if (&L == &rs.L[0] && rs.x.W1s) {   // NFP: each rank updates only its column slice of W^1
        if (rs.x.w_cols > 0 && (st = add(rs.x.W1s, rs.x.dW1s, int64_t(L.d_out) * rs.x.w_cols, rs.x.Wb1s, rs.x.w_cols,
                                         rs.x.ws_pitch)) != APT_OK)
          return st;
      } else if ((st = add(L.W, L.dW, int64_t(L.d_out) * L.d_in, L.Wb, L.d_in, L.wb_pitch)) != APT_OK) {
        return st;
      }
      if ((st = add(L.b, L.db, L.d_out, nullptr, 1, 0)) != APT_OK) return st;
      if (&L == &rs.L[0] && t->gat_heads &&
          ((st = add(rs.ga.a_src, rs.ga.da_src, L.d_out, nullptr, 1, 0)) != APT_OK ||
           (st = add(rs.ga.a_dst, rs.ga.da_dst, L.d_out, nullptr, 1, 0)) != APT_OK))
        return st;
    }
  }
  if (bt.n) {
    CK(c, launch_sgd_multi(bt, t->m.lr, c->stream));
    c->launches++;
  }
  return APT_OK;
}

apt_status compute_body(apt_trainer* t, int update);

// Unpipelined step on sample set q: sampling on the main stream (transposes forked),
// then the compute phases.
apt_status step_body(apt_trainer* t, int update, bool host_batch, int q = 0) {
  apt_ctx* c = t->ctx;
  CK(c, record_ev(t, 0));
  t->csc_forked = false;
  apt_status s = sample_all(t, q, host_batch, c->stream, true);
  if (s != APT_OK) return s;
  activate(t, q);
  t->deferred_fork = nullptr;   // unpipelined: nothing to fork (a failed earlier call may have left one)
  t->pfork_recorded = false;
  return compute_body(t, update);
}

// Pipelined step: compute on set p while the next step (id `next` is the value of the
// set_step node, patched per replay) is sampled into set p^1 on the sampling stream.
// Run the next-step sampling fork now, or leave it for compute_body to launch right
// after the layer-1 forward.
// Fork point 3: the branch is captured after the layer-1 gather (like 2) but from the
// fork event recorded at the step start, so it still depends on nothing of this step.
static apt_status fork_or_defer(apt_trainer* t, std::function<apt_status()> fork) {
  const int fp = sample_fork_point();
  if (fp != 0 && (fp == 1 || (!t->gat_heads && (t->world == 1 || t->s == APT_GDP)))) {
    if (fp == 3) {
      apt_status s = check_cuda(t->ctx, cudaEventRecord(t->ctx->ev_pfork, t->ctx->stream), "fork event");
      if (s != APT_OK) return s;
      t->pfork_recorded = true;
    }
    t->deferred_fork = std::move(fork);
    return APT_OK;
  }
  return fork();
}

// The fork event of the next step's sampling branch (recorded here unless fork point 3
// recorded it at the step start).
static cudaError_t pfork_record(apt_trainer* t) {
  if (t->pfork_recorded) {
    t->pfork_recorded = false;
    return cudaSuccess;
  }
  return cudaEventRecord(t->ctx->ev_pfork, t->ctx->stream);
}

apt_status pipelined_body(apt_trainer* t, int p, int update, uint64_t next) {
  apt_ctx* c = t->ctx;
  CK(c, record_ev(t, 0));
  apt_status s = fork_or_defer(t, [t, c, p, next]() -> apt_status {
    CK(c, pfork_record(t));
    CK(c, cudaStreamWaitEvent(c->samp, c->ev_pfork, 0));
    set_step_kernel<<<1, 1, 0, c->samp>>>(t->step_cells + (p ^ 1), next);
    CK(c, cudaGetLastError());
    c->launches++;
    apt_status s2 = sample_all(t, p ^ 1, false, c->samp, false);
    if (s2 == APT_OK && t->z_prefetch && t->z_where == 1) s2 = prefetch_z(t, p ^ 1, c->samp);   // next batch's layer-1 Z
    if (s2 != APT_OK) return s2;
    if (t->bg_csc_forked) {
      CK(c, cudaEventRecord(c->ev_sjoin, c->samp2));
      CK(c, cudaStreamWaitEvent(c->samp, c->ev_sjoin, 0));
      t->bg_csc_forked = false;
    }
    CK(c, cudaEventRecord(c->ev_pjoin, c->samp));
    return APT_OK;
  });
  if (s != APT_OK) return s;
  t->csc_forked = false;
  activate(t, p);
  t->z_ready = t->z_prefetch;   // this batch's Z was aggregated by the previous step's branch (or the prime)
  t->z_next = (t->z_prefetch && t->z_where == 2) ? (p ^ 1) : -1;
  s = compute_body(t, update);
  t->z_ready = false;
  t->z_next = -1;
  if (s != APT_OK) return s;
  CK(c, cudaStreamWaitEvent(c->stream, c->ev_pjoin, 0));   // next step's batch complete
  return APT_OK;
}

apt_status compute_body(apt_trainer* t, int update) {
  apt_ctx* c = t->ctx;
  const bool gdp = t->world == 1 || t->s == APT_GDP;
  CK(c, record_ev(t, 1));
  if (t->gat_heads) {
    apt_status s = gat_layer1_fwd(t, true);
    if (s == APT_OK) s = hidden1_to_bf16(t);
    if (s != APT_OK) return s;
  } else if (gdp) {
    bool first = true;
    for (auto& rs : t->R) {
      apt_status s = layer1_fwd_gdp(t, rs, first);
      first = false;
      if (s != APT_OK) return s;
    }
  } else {
    apt_status s = layer1_fwd_strategy(t);
    if (s == APT_OK) s = hidden1_to_bf16(t);
    if (s != APT_OK) return s;
  }
  if (t->deferred_fork) {   // pipelined: the next step's sampling branch forks here
    std::function<apt_status()> f = std::move(t->deferred_fork);
    t->deferred_fork = nullptr;
    apt_status s = f();
    if (s != APT_OK) return s;
  }
  CK(c, record_ev(t, 2));
  for (auto& rs : t->R) {
    apt_status s = upper_fwd_loss(t, rs);
    if (s != APT_OK) return s;
  }
  CK(c, record_ev(t, 3));
  // backward (the gradient accumulators were zeroed by the loss kernel)
  for (auto& rs : t->R) {
    apt_status s = upper_bwd(t, rs);
    if (s != APT_OK) return s;
  }
  if (t->z_next >= 0) {
    // the next batch's layer-1 gather+mean beside this step's tail (weight gradient of
    // layer 1, SGD): it needs the next batch's sampling (ev_pjoin) and nothing of this step
    CK(c, cudaEventRecord(t->ev_zt, c->stream));
    CK(c, cudaStreamWaitEvent(c->samp, t->ev_zt, 0));
    CK(c, cudaStreamWaitEvent(c->samp, c->ev_pjoin, 0));
    apt_status s = prefetch_z(t, t->z_next, c->samp);
    if (s != APT_OK) return s;
    CK(c, cudaEventRecord(t->ev_zf, c->samp));
  }
  if (t->gat_heads) {
    apt_status s = gat_layer1_bwd(t);
    if (s != APT_OK) return s;
  } else if (gdp) {
    for (auto& rs : t->R) {
      apt_status s = layer1_bwd_gdp(t, rs);
      if (s != APT_OK) return s;
    }
  } else {
    apt_status s = layer1_bwd_strategy(t);
    if (s != APT_OK) return s;
  }
  if (t->K > 1) {   // join the weight-gradient branch forked in upper_bwd
    CK(c, cudaEventRecord(c->ev_join, c->side));
    CK(c, cudaStreamWaitEvent(c->stream, c->ev_join, 0));
  }
  CK(c, record_ev(t, 4));
  apt_status s = allreduce_sgd(t, update);
  if (s != APT_OK) return s;
  if (t->z_next >= 0) CK(c, cudaStreamWaitEvent(c->stream, t->ev_zf, 0));   // the next step's Z is ready
  CK(c, record_ev(t, 5));
  t->ev_ok = true;
  return APT_OK;
}

// The layer-1 forward on the active sample set (every hosted rank): GAT, GDP, or the
// strategy's Permute/Shuffle/Execute/Reshuffle; h^1 left in L[0].H / Hb.
apt_status layer1_forward(apt_trainer* t) {
  apt_status s = APT_OK;
  if (t->gat_heads) {
    s = gat_layer1_fwd(t, false);
    return s == APT_OK ? hidden1_to_bf16(t) : s;
  }
  if (t->world == 1 || t->s == APT_GDP) {
    bool first = true;
    for (auto& rs : t->R) {
      s = layer1_fwd_gdp(t, rs, first);
      first = false;
      if (s != APT_OK) return s;
    }
    return APT_OK;
  }
  s = layer1_fwd_strategy(t);
  return s == APT_OK ? hidden1_to_bf16(t) : s;
}

// rows [0, n) of a bf16 or fp32 matrix -> fp32 rows of `dp` floats (layer API outputs)
__global__ void rows_to_f32_kernel(float* __restrict__ dst, int64_t dp, const float* __restrict__ src,
                                   const uint16_t* __restrict__ srcb, int64_t sp, int cols, int64_t n) {
  const int64_t total = n * cols;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = i / cols;
    const int c = int(i - r * cols);
    dst[r * dp + c] = srcb ? bf16_bits_to_float(srcb[r * sp + c]) : src[r * sp + c];
  }
}

}  // namespace apt

// A first-layer session of the standalone layer API (apt_layer_fwd / apt_layer_bwd,
// SURVEY §8(b)): an internal layer-only trainer whose layer-1 hop holds the caller's
// sampled blocks, and the row layout of h1 / dh1 (hosted ranks concatenated in order).
struct apt_layer_saved {
  apt_ctx* ctx = nullptr;
  apt_trainer* t = nullptr;
  int n_local = 0;
  int64_t rows[APT_MAX_RANKS] = {};
  int64_t off[APT_MAX_RANKS + 1] = {};
  int d_in = 0, d_out = 0;
};

extern "C" {

apt_status apt_layer_saved_destroy(apt_layer_saved* sv) {
  if (!sv) return APT_OK;
  apt_ctx* c = sv->ctx;
  if (sv->t) apt_trainer_destroy(sv->t);
  delete sv;
  if (c) ctx_release(c);
  return APT_OK;
}

apt_status apt_layer_fwd(apt_ctx* c, apt_strategy s, const apt_batch* batch, const apt_fstore* f, const float* W,
                         const float* bias, int d_out, apt_dtype dtype, float* h1_out, apt_layer_saved** saved) {
  if (!c || !batch || !f || !W || !bias || !h1_out || !saved || d_out < 1 || s < APT_GDP || s > APT_DNP)
    return set_err(c, APT_E_INVALID, "apt_layer_fwd: bad arguments (batch %p store %p W %p bias %p h1 %p saved %p "
                                     "d_out %d strategy %d)", (const void*)batch, (const void*)f, (const void*)W,
                   (const void*)bias, (const void*)h1_out, (const void*)saved, d_out, int(s));
  if (c->broken) return set_err(c, APT_E_STATE, "ctx is broken by an earlier CUDA error");
  if (batch->ctx != c || f->ctx != c) return set_err(c, APT_E_INVALID, "apt_layer_fwd: batch / store of another ctx");
  if ((dtype == APT_BF16) != (f->dtype == kBF16)) return set_err(c, APT_E_INVALID, "apt_layer_fwd: dtype != store dtype");
  std::vector<const apt_batch*> per;
  if (batch->members.empty()) per.push_back(batch);
  else per = batch->members;
  if (int(per.size()) != c->n_local)
    return set_err(c, APT_E_INVALID, "apt_layer_fwd: %zu batches for %d hosted ranks (apt_batch_group)", per.size(),
                   c->n_local);
  if (batch->g != f->g) return set_err(c, APT_E_INVALID, "apt_layer_fwd: batch and store are on different graphs");
  const int K = batch->K;
  apt_model_desc m{};
  m.n_layers = K;
  m.dims[0] = f->dim;
  m.dims[1] = d_out;
  for (int l = 2; l <= K; ++l) m.dims[l] = 8;          // upper layers unused by a layer session
  int64_t B = 1;
  for (auto* b : per) B = std::max<int64_t>(B, b->n_dst[0]);
  for (int l = 0; l < K; ++l) m.fanouts[l] = batch->fanouts[l];
  m.batch = int(B);
  m.dtype = dtype;
  m.sample_seed = batch->rng_seed;                      // owners re-sample with the batch's key (R1)
  auto* sv = new apt_layer_saved();
  sv->ctx = c;
  ctx_retain(c);
  sv->n_local = c->n_local;
  sv->d_in = f->dim;
  sv->d_out = d_out;
  apt_status st = trainer_create(c, batch->g, f, &m, s, nullptr, &sv->t, true);
  if (st != APT_OK) { apt_layer_saved_destroy(sv); return st; }
  apt_trainer* t = sv->t;
  if ((st = apt_trainer_set_params(t, 1, W, bias)) != APT_OK) { apt_layer_saved_destroy(sv); return st; }
  const uint64_t step = batch->step;
  CK(c, cudaMemcpyAsync(t->step_cells, &step, sizeof(step), cudaMemcpyHostToDevice, c->stream));
  // the caller's layer-1 blocks (hop K-1, sampler ELL form) into sample set 0 of every rank
  for (int li = 0; li < c->n_local; ++li) {
    const apt_batch* b = per[li];
    Hop& hp = t->R[li].sset[0].hops[K - 1];
    const int64_t n = b->n_dst[K - 1];
    if (n > hp.max_dst) { apt_layer_saved_destroy(sv); return set_err(c, APT_E_INVALID, "apt_layer_fwd: block too large"); }
    CK(c, cudaMemcpyAsync(const_cast<int32_t*>(hp.dst), b->dst[K - 1], sizeof(int32_t) * n, cudaMemcpyDeviceToDevice,
                          c->stream));
    const int32_t n32 = int32_t(n);
    CK(c, cudaMemcpyAsync(const_cast<int32_t*>(hp.n_dst), &n32, 4, cudaMemcpyHostToDevice, c->stream));
    CK(c, cudaMemcpyAsync(hp.cnt, b->cnt[K - 1], sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, c->stream));
    CK(c, cudaMemcpyAsync(hp.nbr, b->nbr[K - 1], sizeof(int32_t) * n * hp.k, cudaMemcpyDeviceToDevice, c->stream));
    sv->rows[li] = n;
    sv->off[li + 1] = sv->off[li] + n;
  }
  CK(c, cudaStreamSynchronize(c->stream));   // host staging of the counts above
  t->primed = -1;
  activate(t, 0);
  if ((st = layer1_forward(t)) != APT_OK) { apt_layer_saved_destroy(sv); return st; }
  for (int li = 0; li < c->n_local; ++li) {
    const Layer& L = t->R[li].L[0];
    if (!sv->rows[li]) continue;
    rows_to_f32_kernel<<<unsigned(blocks_for(sv->rows[li] * d_out)), 256, 0, c->stream>>>(
        h1_out + sv->off[li] * d_out, d_out, L.H, L.Hb, L.Hb ? L.hb_pitch : L.h_pitch, d_out, sv->rows[li]);
    CK(c, cudaGetLastError());
    c->launches++;
  }
  *saved = sv;
  return APT_OK;
}

apt_status apt_layer_bwd(apt_ctx* c, apt_layer_saved* sv, const float* dh1, float* dW, float* dbias) {
  if (!c || !sv || sv->ctx != c || !dh1 || !dW || !dbias) return set_err(c, APT_E_INVALID, "apt_layer_bwd: bad arguments");
  apt_trainer* t = sv->t;
  std::vector<const float*> ptr(sv->n_local);
  for (int li = 0; li < sv->n_local; ++li) ptr[li] = dh1 + sv->off[li] * sv->d_out;
  apt_status st = apt_trainer_layer_bwd(t, ptr.data(), sv->d_out);
  if (st != APT_OK) return st;
  const RankState& r0 = t->R[0];
  const Layer& L = r0.L[0];
  if (r0.x.dW1s) {   // NFP: W^1 is column-owned -- the hosted ranks' slices into their columns
    for (auto& rs : t->R)
      if (rs.x.w_cols > 0)
        CK(c, cudaMemcpy2DAsync(dW + rs.x.col_lo, sizeof(float) * L.d_in, rs.x.dW1s, sizeof(float) * rs.x.w_cols,
                                sizeof(float) * rs.x.w_cols, L.d_out, cudaMemcpyDeviceToDevice, c->stream));
  } else {
    CK(c, cudaMemcpyAsync(dW, L.dW, sizeof(float) * L.d_out * L.d_in, cudaMemcpyDeviceToDevice, c->stream));
  }
  CK(c, cudaMemcpyAsync(dbias, L.db, sizeof(float) * L.d_out, cudaMemcpyDeviceToDevice, c->stream));
  return APT_OK;
}

// ---- the first layer alone (the part APT parallelises), bound to a trainer:
// the trainer samples step `step` of its epoch, then runs the layer-1 forward ...
apt_status apt_trainer_layer_fwd(apt_trainer* t, int64_t step) {
  if (!t || !t->perm) return set_err(t ? t->ctx : nullptr, APT_E_STATE, "apt_trainer_layer_fwd: call apt_trainer_set_epoch first");
  apt_ctx* c = t->ctx;
  if (c->broken) return set_err(c, APT_E_STATE, "ctx is broken by an earlier CUDA error");
  t->primed = -1;   // sample set 0 is overwritten
  t->host_primed = false;
  set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells, uint64_t(step));
  CK(c, cudaGetLastError());
  c->launches++;
  t->csc_forked = false;
  {
    apt_status s = sample_all(t, 0, false, c->stream, false);
    if (s != APT_OK) return s;
  }
  activate(t, 0);
  return layer1_forward(t);
}

// ... and backward from dL/dh1 (one device pointer per hosted rank, rows of the
// rank's layer-1 destinations, fp32, `pitch` floats apart): dW1/db1 of the
// strategy, all-reduced over the ranks (NFP: column-owned slices).
apt_status apt_trainer_layer_bwd(apt_trainer* t, const float* const* dh1, int64_t pitch) {
  if (!t || !dh1 || pitch < t->m.dims[1]) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "apt_trainer_layer_bwd: bad arguments");
  apt_ctx* c = t->ctx;
  const bool bf = t->m.dtype == APT_BF16;
  const int relu = t->K > 1 ? 1 : 0;
  for (size_t li = 0; li < t->R.size(); ++li) {
    RankState& rs = t->R[li];
    Layer& L = rs.L[0];
    if (!dh1[li]) return set_err(c, APT_E_INVALID, "apt_trainer_layer_bwd: dh1[%zu] is null", li);
    // G = dh1 (copied over the rows the step produced; the count stays on the device)
    launch_pdl(copy_rows_kernel, dim3(blocks_for(L.max_rows * L.d_out)), dim3(256), 0, c->stream, L.G, L.h_pitch, dh1[li], pitch, L.d_out,
                                                                             L.n_rows);
    CK(c, cudaGetLastError());
    if (bf) CK(c, launch_grad_finish(L.G, L.h_pitch, L.H, L.h_pitch, L.d_out, relu, L.Gb, L.gb_pitch, L.n_rows,
                                     L.max_rows, c->stream, L.Hb, L.hb_pitch));
    else if (relu) CK(c, launch_relu_bwd(L.G, L.H, L.h_pitch, L.d_out, L.n_rows, L.max_rows, c->stream));
    CK(c, cudaMemsetAsync(L.dW, 0, sizeof(float) * grad_floats_l1(t), c->stream));
    c->launches++;
  }
  if (t->gat_heads) {
    apt_status s = gat_layer1_bwd(t);
    if (s != APT_OK) return s;
  } else if (t->world == 1 || t->s == APT_GDP) {
    for (auto& rs : t->R) {
      apt_status s = layer1_bwd_gdp(t, rs);
      if (s != APT_OK) return s;
    }
  } else {
    apt_status s = layer1_bwd_strategy(t);
    if (s != APT_OK) return s;
  }
  if (t->world > 1) return allreduce_grads(t, grad_floats_l1(t));
  return APT_OK;
}

apt_status apt_trainer_step(apt_trainer* t, int64_t step, int update) {
  if (!t || !t->perm) return set_err(t ? t->ctx : nullptr, APT_E_STATE, "apt_trainer_step: call apt_trainer_set_epoch first");
  apt_ctx* c = t->ctx;
  if (c->broken) return set_err(c, APT_E_STATE, "ctx is broken by an earlier CUDA error");
  update = update ? 1 : 0;
  t->host_primed = false;   // the host-batch pipeline's prefetched set may be overwritten
  if (!t->pipeline) {
    // one stream: sampling, then compute, on sample set 0
    t->primed = -1;
    if (t->use_graph) {
      if (!t->gexec || t->graph_update != update) {
        if (t->gexec) { cudaGraphExecDestroy(t->gexec); t->gexec = nullptr; }
        if (t->graph) { cudaGraphDestroy(t->graph); t->graph = nullptr; }
        cudaGraph_t graph;
        CK(c, cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal));
        set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells, uint64_t(step));
        const int64_t l0 = c->launches;
        t->capturing = true;
        apt_status s = step_body(t, update, false, 0);
        t->capturing = false;
        const cudaError_t ej = s == APT_OK ? tap_join(t) : cudaSuccess;
        t->tapped = false;
        cudaError_t e = cudaStreamEndCapture(c->stream, &graph);
        if (e == cudaSuccess) e = ej;
        t->launches_per_step = c->launches - l0 + 1;   // counted at replay, not at capture
        c->launches = l0;
        if (s != APT_OK) return s;
        CK(c, e);
        t->step_node = find_step_node(graph);
        if (!t->step_node) { cudaGraphDestroy(graph); return set_err(c, APT_E_CUDA, "step node not found in graph"); }
        CK(c, cudaGraphInstantiate(&t->gexec, graph, 0));
        t->graph = graph;
        t->graph_update = update;
      }
      CK(c, patch_step_node(t->gexec, t->step_node, t->step_cells, uint64_t(step)));
      CK(c, cudaGraphLaunch(t->gexec, c->stream));
      c->launches += t->launches_per_step;
      return APT_OK;
    }
    set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells, uint64_t(step));
    CK(c, cudaGetLastError());
    c->launches++;
    return step_body(t, update, false, 0);
  }
  // pipelined: this step's batch was sampled during the previous step (else sample it now)
  int p;
  if (t->primed == step) {
    p = t->primed_parity;
  } else {
    p = t->parity ^ 1;
    set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells + p, uint64_t(step));
    CK(c, cudaGetLastError());
    c->launches++;
    t->csc_forked = false;
    apt_status s = sample_all(t, p, false, c->stream, false);
    if (s == APT_OK && t->z_prefetch) s = prefetch_z(t, p, c->stream);
    if (s != APT_OK) return s;
  }
  const uint64_t next = uint64_t(step + 1);
  if (t->use_graph) {
    if (!t->gexec_p[p][update]) {
      cudaGraph_t graph;
      CK(c, cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal));
      const int64_t l0 = c->launches;
      t->capturing = true;
      apt_status s = pipelined_body(t, p, update, next);
      t->capturing = false;
      const cudaError_t ej = s == APT_OK ? tap_join(t) : cudaSuccess;
      t->tapped = false;
      cudaError_t e = cudaStreamEndCapture(c->stream, &graph);
      if (e == cudaSuccess) e = ej;
      t->launches_p[p][update] = c->launches - l0;
      c->launches = l0;
      if (s != APT_OK) return s;
      CK(c, e);
      t->step_node_p[p][update] = find_step_node(graph);
      if (!t->step_node_p[p][update]) { cudaGraphDestroy(graph); return set_err(c, APT_E_CUDA, "step node not found in graph"); }
      CK(c, cudaGraphInstantiate(&t->gexec_p[p][update], graph, 0));
      t->graph_p[p][update] = graph;
    }
    activate(t, p);   // readouts after the step see the computed set
    CK(c, patch_step_node(t->gexec_p[p][update], t->step_node_p[p][update], t->step_cells + (p ^ 1), next));
    CK(c, cudaGraphLaunch(t->gexec_p[p][update], c->stream));
    c->launches += t->launches_p[p][update];
  } else {
    apt_status s = pipelined_body(t, p, update, next);
    if (s != APT_OK) return s;
  }
  t->primed = step + 1;
  t->primed_parity = p ^ 1;
  return APT_OK;
}

apt_status apt_trainer_set_pipeline(apt_trainer* t, int enable) {
  if (!t) return set_err(nullptr, APT_E_INVALID, "null trainer");
  t->pipeline = enable != 0;
  t->primed = -1;
  return APT_OK;
}

apt_status apt_trainer_step_host(apt_trainer* t, const int64_t* gbatch, int64_t n_global, int64_t step, int update,
                                 float* loss_host) {
  if (!t || !gbatch || !loss_host || n_global < 1 || n_global > int64_t(t->world) * t->m.batch)
    return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "apt_trainer_step_host: bad arguments");
  apt_ctx* c = t->ctx;
  if (c->broken) return set_err(c, APT_E_STATE, "ctx is broken by an earlier CUDA error");
  // the global batch into pinned staging ([n, ids...], int32); ranks pick their seeds on
  // the device.  The previous call ended with a sync, so the staging is free.
  t->hb_pinned[0] = int32_t(n_global);
  for (int64_t i = 0; i < n_global; ++i) {
    const int64_t u = gbatch[i];
    if (u < 0 || u >= t->g->n) return set_err(c, APT_E_INVALID, "step_host: seed %lld out of range", (long long)u);
    t->hb_pinned[1 + i] = int32_t(u);
  }
  const size_t hb_bytes = sizeof(int32_t) * size_t(t->hb_len);
  t->primed = -1;   // sample set 0 is overwritten
  t->host_primed = false;
  // H2D batch -> step -> D2H per-rank losses, one stream-ordered sequence (one graph replay)
  auto body = [&]() -> apt_status {
    CK(c, cudaMemcpyAsync(t->hb_dev, t->hb_pinned, hb_bytes, cudaMemcpyHostToDevice, c->stream));
    set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells, uint64_t(step));
    CK(c, cudaGetLastError());
    apt_status s = step_body(t, update, true);
    if (s != APT_OK) return s;
    for (size_t i = 0; i < t->R.size(); ++i)
      CK(c, cudaMemcpyAsync(t->loss_pinned + i, t->R[i].loss, sizeof(float), cudaMemcpyDeviceToHost, c->stream));
    return APT_OK;
  };
  if (t->use_graph) {
    if (!t->gexec_host || t->graph_host_update != update) {
      if (t->gexec_host) { cudaGraphExecDestroy(t->gexec_host); t->gexec_host = nullptr; }
      if (t->graph_host) { cudaGraphDestroy(t->graph_host); t->graph_host = nullptr; }
      cudaGraph_t graph;
      CK(c, cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal));
      const int64_t l0 = c->launches;
      t->capturing = true;
      apt_status s = body();
      t->capturing = false;
      const cudaError_t ej = s == APT_OK ? tap_join(t) : cudaSuccess;
      t->tapped = false;
      cudaError_t e = cudaStreamEndCapture(c->stream, &graph);
      if (e == cudaSuccess) e = ej;
      const int64_t per = c->launches - l0 + 1;
      c->launches = l0;
      if (s != APT_OK) return s;
      CK(c, e);
      t->step_node_host = find_step_node(graph);
      if (!t->step_node_host) { cudaGraphDestroy(graph); return set_err(c, APT_E_CUDA, "step node not found in graph"); }
      CK(c, cudaGraphInstantiate(&t->gexec_host, graph, 0));
      t->graph_host = graph;
      t->graph_host_update = update;
      t->launches_per_step_host = per;
    }
    CK(c, patch_step_node(t->gexec_host, t->step_node_host, t->step_cells, uint64_t(step)));
    CK(c, cudaGraphLaunch(t->gexec_host, c->stream));
    c->launches += t->launches_per_step_host;
  } else {
    apt_status s = body();
    if (s != APT_OK) return s;
    c->launches++;
  }
  CK(c, cudaStreamSynchronize(c->stream));
  float tot = 0.f;
  for (size_t i = 0; i < t->R.size(); ++i) tot += t->loss_pinned[i];
  *loss_host = tot;
  return apt_ctx_sync(c);
}

// Pipelined end-to-end call: submit the NEXT global batch (host, copied to pinned
// staging) and run the step of the batch submitted by the previous call; returns that
// step's loss.  While the step computes, the next batch is copied in and sampled on
// the sampling stream (one graph replay per call).  The first call only primes (loss
// NaN, *had_step = 0).
static apt_status step_host_pipelined_impl(apt_trainer* t, const int64_t* next_batch, int64_t n_next, int64_t next_step,
                                           int update, float* loss_prev, int* had_step, bool async) {
  if (!t || !next_batch || !loss_prev || !had_step || n_next < 1 || n_next > int64_t(t->world) * t->m.batch)
    return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "apt_trainer_step_host_pipelined: bad arguments");
  apt_ctx* c = t->ctx;
  if (c->broken) return set_err(c, APT_E_STATE, "ctx is broken by an earlier CUDA error");
  update = update ? 1 : 0;
  t->primed = -1;
  const int p = t->host_primed ? t->host_parity : 0;   // set holding the batch to compute
  const int q = t->host_primed ? p ^ 1 : 0;            // set receiving the next batch
  int32_t* stage = t->hb_pinned + q * t->hb_len;
  stage[0] = int32_t(n_next);
  for (int64_t i = 0; i < n_next; ++i) {
    const int64_t u = next_batch[i];
    if (u < 0 || u >= t->g->n) return set_err(c, APT_E_INVALID, "step_host: seed %lld out of range", (long long)u);
    stage[1 + i] = int32_t(u);
  }
  const size_t hb_bytes = sizeof(int32_t) * size_t(t->hb_len);
  if (!t->host_primed) {   // prime: copy in and sample the first batch into set 0
    t->async_pending = false;
    CK(c, cudaMemcpyAsync(t->hb_dev, stage, hb_bytes, cudaMemcpyHostToDevice, c->stream));
    set_step_kernel<<<1, 1, 0, c->stream>>>(t->step_cells, uint64_t(next_step));
    CK(c, cudaGetLastError());
    t->csc_forked = false;
    apt_status s = sample_all(t, 0, true, c->stream, false);
    if (s == APT_OK && t->z_prefetch) s = prefetch_z(t, 0, c->stream);
    if (s != APT_OK) return s;
    CK(c, cudaStreamSynchronize(c->stream));
    t->host_primed = true;
    t->host_parity = 0;
    *loss_prev = std::nanf("");
    *had_step = 0;
    return apt_ctx_sync(c);
  }
  auto body = [&](uint64_t nstep) -> apt_status {
    CK(c, record_ev(t, 0));
    apt_status s = fork_or_defer(t, [&, nstep]() -> apt_status {
      CK(c, pfork_record(t));
      CK(c, cudaStreamWaitEvent(c->samp, c->ev_pfork, 0));
      CK(c, cudaMemcpyAsync(t->hb_dev + q * t->hb_len, stage, hb_bytes, cudaMemcpyHostToDevice, c->samp));
      set_step_kernel<<<1, 1, 0, c->samp>>>(t->step_cells + q, nstep);
      CK(c, cudaGetLastError());
      apt_status s2 = sample_all(t, q, true, c->samp, false);
      if (s2 == APT_OK && t->z_prefetch && t->z_where == 1) s2 = prefetch_z(t, q, c->samp);
      if (s2 != APT_OK) return s2;
      if (t->bg_csc_forked) {
        CK(c, cudaEventRecord(c->ev_sjoin, c->samp2));
        CK(c, cudaStreamWaitEvent(c->samp, c->ev_sjoin, 0));
        t->bg_csc_forked = false;
      }
      CK(c, cudaEventRecord(c->ev_pjoin, c->samp));
      return APT_OK;
    });
    if (s != APT_OK) return s;
    t->csc_forked = false;
    activate(t, p);
    t->z_ready = t->z_prefetch;
    t->z_next = (t->z_prefetch && t->z_where == 2) ? q : -1;
    s = compute_body(t, update);
    t->z_ready = false;
    t->z_next = -1;
    if (s != APT_OK) return s;
    for (size_t i = 0; i < t->R.size(); ++i)
      CK(c, cudaMemcpyAsync(t->loss_pinned + p * APT_MAX_RANKS + i, t->R[i].loss, sizeof(float),
                            cudaMemcpyDeviceToHost, c->stream));
    CK(c, cudaStreamWaitEvent(c->stream, c->ev_pjoin, 0));
    return APT_OK;
  };
  if (t->use_graph) {
    if (!t->gexec_hp[p][update]) {
      cudaGraph_t graph;
      CK(c, cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal));
      const int64_t l0 = c->launches;
      t->capturing = true;
      apt_status s = body(uint64_t(next_step));
      t->capturing = false;
      const cudaError_t ej = s == APT_OK ? tap_join(t) : cudaSuccess;
      t->tapped = false;
      cudaError_t e = cudaStreamEndCapture(c->stream, &graph);
      if (e == cudaSuccess) e = ej;
      t->launches_hp[p][update] = c->launches - l0 + 1;
      c->launches = l0;
      if (s != APT_OK) return s;
      CK(c, e);
      t->step_node_hp[p][update] = find_step_node(graph);
      if (!t->step_node_hp[p][update]) { cudaGraphDestroy(graph); return set_err(c, APT_E_CUDA, "step node not found"); }
      CK(c, cudaGraphInstantiate(&t->gexec_hp[p][update], graph, 0));
      t->graph_hp[p][update] = graph;
    }
    activate(t, p);
    CK(c, patch_step_node(t->gexec_hp[p][update], t->step_node_hp[p][update], t->step_cells + q, uint64_t(next_step)));
    CK(c, cudaGraphLaunch(t->gexec_hp[p][update], c->stream));
    c->launches += t->launches_hp[p][update];
  } else {
    apt_status s = body(uint64_t(next_step));
    if (s != APT_OK) return s;
    c->launches++;
  }
  t->host_parity = q;
  if (async) {
    // the step just launched keeps the device busy while the host returns the loss of the
    // step the PREVIOUS call launched (its loss slot is the other parity)
    CK(c, cudaEventRecord(t->ev_done[p], c->stream));
    *had_step = 0;
    if (t->async_pending) {
      CK(c, cudaEventSynchronize(t->ev_done[p ^ 1]));
      float tot = 0.f;
      for (size_t i = 0; i < t->R.size(); ++i) tot += t->loss_pinned[(p ^ 1) * APT_MAX_RANKS + i];
      *loss_prev = tot;
      *had_step = 1;
    }
    t->async_pending = true;
    CK(c, cudaGetLastError());
    return APT_OK;
  }
  t->async_pending = false;
  CK(c, cudaStreamSynchronize(c->stream));
  float tot = 0.f;
  for (size_t i = 0; i < t->R.size(); ++i) tot += t->loss_pinned[p * APT_MAX_RANKS + i];
  *loss_prev = tot;
  *had_step = 1;
  return apt_ctx_sync(c);
}

apt_status apt_trainer_step_host_pipelined(apt_trainer* t, const int64_t* next_batch, int64_t n_next, int64_t next_step,
                                           int update, float* loss_prev, int* had_step) {
  return step_host_pipelined_impl(t, next_batch, n_next, next_step, update, loss_prev, had_step, false);
}

apt_status apt_trainer_step_host_async(apt_trainer* t, const int64_t* next_batch, int64_t n_next, int64_t next_step,
                                       int update, float* loss_prev, int* had_step) {
  return step_host_pipelined_impl(t, next_batch, n_next, next_step, update, loss_prev, had_step, true);
}

apt_status apt_trainer_loss(apt_trainer* t, float* loss) {
  if (!t || !loss) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "loss: null");
  apt_ctx* c = t->ctx;
  float tot = 0.f;
  for (auto& rs : t->R) {
    float v = 0.f;
    CK(c, cudaMemcpyAsync(&v, rs.loss, 4, cudaMemcpyDeviceToHost, c->stream));
    CK(c, cudaStreamSynchronize(c->stream));
    tot += v;
  }
  *loss = tot;
  return apt_ctx_sync(c);
}

apt_status apt_trainer_use_graph(apt_trainer* t, int enable) {
  if (!t) return set_err(nullptr, APT_E_INVALID, "null trainer");
  t->use_graph = enable != 0;
  return APT_OK;
}

apt_status apt_trainer_phase_ms(apt_trainer* t, double* ms, int n) {
  if (!t || !ms || n < 1) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "phase_ms: bad args");
  CK(t->ctx, cudaStreamSynchronize(t->ctx->stream));
  if (!t->ev_ok) return set_err(t->ctx, APT_E_STATE, "phase_ms: no step recorded");
  for (int i = 0; i < n && i < 6; ++i) {
    float v = 0.f;
    if (i < 5) CK(t->ctx, cudaEventElapsedTime(&v, t->ev[i], t->ev[i + 1]));
    else CK(t->ctx, cudaEventElapsedTime(&v, t->ev[6], t->ev[7]));
    ms[i] = v;
  }
  return APT_OK;
}

apt_status apt_trainer_read(apt_trainer* t, int rank, int what, int layer, void* host, int64_t cap, int64_t* rows,
                            int* cols) {
  if (!t || !host || !rows || !cols) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "read: null");
  apt_ctx* c = t->ctx;
  RankState* rs = nullptr;
  for (auto& r : t->R)
    if (r.rank == rank) rs = &r;
  if (!rs) return set_err(c, APT_E_INVALID, "read: rank %d not hosted", rank);
  if (what != 0 && (layer < 1 || layer > t->K)) return set_err(c, APT_E_INVALID, "read: layer out of range");
  CK(c, cudaStreamSynchronize(c->stream));
  auto count = [&](const int32_t* p) {
    int32_t v = 0;
    cudaMemcpy(&v, p, 4, cudaMemcpyDeviceToHost);
    return int64_t(v);
  };
  auto copy_rows = [&](const void* src, int64_t nr, int nc, int64_t pitch, int esz, bool bf) -> apt_status {
    *rows = nr;
    *cols = nc;
    const int64_t n = std::min<int64_t>(cap, nr * nc);
    std::vector<uint8_t> buf(size_t(std::max<int64_t>(nr, 1) * pitch * esz));
    if (nr) CK(c, cudaMemcpy(buf.data(), src, size_t(nr * pitch * esz), cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < n; ++i) {
      const int64_t r = i / nc, cc = i % nc;
      if (bf) {
        uint32_t b = uint32_t(reinterpret_cast<uint16_t*>(buf.data())[r * pitch + cc]) << 16;
        memcpy(static_cast<float*>(host) + i, &b, 4);
      } else if (esz == 4) {
        memcpy(static_cast<uint8_t*>(host) + i * 4, buf.data() + (r * pitch + cc) * 4, 4);
      }
    }
    return APT_OK;
  };
  switch (what) {
    case 0: return copy_rows(rs->seeds, count(rs->small), 1, 1, 4, false);
    case 1: {
      const Hop& hp = rs->hops[t->K - layer];
      return copy_rows(hp.dst, count(hp.n_dst), 1, 1, 4, false);
    }
    case 2: {
      const Layer& L = rs->L[layer - 1];
      const int64_t nr = count(L.n_rows);
      if (L.Zb) return copy_rows(L.Zb, nr, L.d_in, L.zb_pitch, 2, true);
      return copy_rows(L.Zf, nr, L.d_in, L.zf_pitch, 4, false);
    }
    case 3: {   // bf16 mode, hidden layers: the stored bf16 activation (reading R11)
      const Layer& L = rs->L[layer - 1];
      if (L.Hb) return copy_rows(L.Hb, count(L.n_rows), L.d_out, L.hb_pitch, 2, true);
      return copy_rows(L.H, count(L.n_rows), L.d_out, L.h_pitch, 4, false);
    }
    case 4: {
      const Layer& L = rs->L[layer - 1];
      if (layer == 1 && rs->x.dW1s) {   // NFP: concatenate the column-owned slices of the hosted ranks
        *rows = L.d_out;
        *cols = L.d_in;
        std::vector<float> full(size_t(L.d_out) * L.d_in, 0.f);
        for (auto& o : t->R) {
          if (o.x.w_cols <= 0) continue;
          CK(c, cudaMemcpy2D(full.data() + o.x.col_lo, sizeof(float) * L.d_in, o.x.dW1s, sizeof(float) * o.x.w_cols,
                             sizeof(float) * o.x.w_cols, L.d_out, cudaMemcpyDeviceToHost));
        }
        memcpy(host, full.data(), sizeof(float) * std::min<int64_t>(cap, int64_t(full.size())));
        return APT_OK;
      }
      return copy_rows(L.dW, L.d_out, L.d_in, L.d_in, 4, false);
    }
    case 5: { const Layer& L = rs->L[layer - 1]; return copy_rows(L.db, 1, L.d_out, L.d_out, 4, false); }
    case 6: { const Layer& L = rs->L[layer - 1]; return copy_rows(L.G, count(L.n_rows), L.d_out, L.h_pitch, 4, false); }
    case 7: {   // GAT layer 1: [da_src | da_dst]
      if (!t->gat_heads || layer != 1) return set_err(c, APT_E_INVALID, "read: no attention gradients (GAT layer 1 only)");
      return copy_rows(rs->ga.da_src, 1, 2 * rs->L[0].d_out, 2 * rs->L[0].d_out, 4, false);
    }
    default: return set_err(c, APT_E_INVALID, "read: unknown item %d", what);
  }
}

apt_status apt_trainer_agg_bytes(apt_trainer* t, double* bytes) {
  if (!t || !bytes) return set_err(nullptr, APT_E_INVALID, "agg_bytes: null");
  *bytes = t->last_agg_bytes;
  return APT_OK;
}

}  // extern "C"
