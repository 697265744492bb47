// trainer.h -- per-rank state of the training step (internal).
#pragma once
#include <cuda_runtime.h>

#include <functional>
#include <vector>

#include "runtime.h"

namespace apt {

struct Hop {
  int k = 0;
  int64_t max_dst = 0, max_src = 0;
  const int32_t* dst = nullptr;     // frontier (seeds or previous hop's src)
  const int32_t* n_dst = nullptr;   // device count
  int32_t* cnt = nullptr;           // [max_dst]
  int32_t* nbr = nullptr;           // [max_dst * k] global ids (ELL)
  int32_t* src = nullptr;           // [max_src]
  int32_t* indptr = nullptr;        // [max_dst + 1]
  int32_t* indices = nullptr;       // [max_dst * k]
  int32_t* counts = nullptr;        // [0] n_src, [1] n_edges, [2] csc total
  int32_t* part2 = nullptr;         // scan workspace
  // transpose of the block (upper hops only): in-edges of every local source
  int32_t* csc_cnt = nullptr;       // [max_src] (zero between uses)
  int32_t* csc_ptr = nullptr;       // [max_src + 1]
  int2* csc_dst = nullptr;          // [max_dst * k]
  int32_t* csc_ws = nullptr;        // scan workspace
};

struct Layer {
  int d_in = 0, d_out = 0;
  int64_t zf_pitch = 0, zb_pitch = 0, h_pitch = 0, wb_pitch = 0;
  int64_t max_rows = 0;
  const int32_t* n_rows = nullptr;  // device count of dst rows
  float* Zf = nullptr;              // [max_rows x zf_pitch] (fp32 mode)
  uint16_t* Zb = nullptr;           // [max_rows x zb_pitch] (bf16 mode)
  float* H = nullptr;               // post-activation (or logits)
  uint16_t* Hb = nullptr;           // bf16 mode, hidden layers: the activation as the next layer and the
  int64_t hb_pitch = 0;             //   backward read it (reading R11); GDP projections write only Hb
  float* G = nullptr;               // dL/dpre
  uint16_t* Gb = nullptr;           // bf16 copy of G (tcgen05 backward, bf16 mode)
  uint16_t* Mk = nullptr;           // ReLU mask bits of H (bf16 mode, hidden layers) [max_rows x mk_pitch]
  int64_t mk_pitch = 0;
  mutable bool mk_valid = false;    // the captured forward writes Mk (tcgen05 bf16 epilogue on this rank)
  int64_t gb_pitch = 0;
  float* dZ = nullptr;              // [max_rows x zf_pitch] scratch (l > 1)
  uint16_t* dZb = nullptr;          // bf16 mode: (G W) / deg in bf16 [max_rows x dzb_pitch] (reading R13)
  int64_t dzb_pitch = 0;
  float* W = nullptr;               // [d_out x d_in] fp32 master
  float* b = nullptr;
  uint16_t* Wb = nullptr;           // [d_out x wb_pitch] bf16 copy (tensor cores)
  float* dW = nullptr;
  float* db = nullptr;
};

// NFP / SNP / DNP state of one rank (strategies.cu).  The rank is both a
// requester (its own layer-1 rows, whose h^1 it needs) and an owner (work items
// other ranks -- and itself -- send it: Permute/Shuffle).
struct Xchg {
  int64_t wcap = 0;                  // work-item capacity (sum of all requesters' layer-1 rows)
  int32_t* n_work = nullptr;         // [1] device count of items owned
  int32_t* work_rank = nullptr;      // [wcap] requester rank
  int32_t* work_row = nullptr;       // [wcap] requester layer-1 row
  int32_t* work_gid = nullptr;       // [wcap] destination node id
  int32_t* wcnt = nullptr;           // [wcap] re-sampled ELL count (same Philox key: identical sample)
  int32_t* wnbr = nullptr;           // [wcap * k]
  int w_cols = 0;                    // aggregated columns: d, or the NFP column slice width
  int64_t wzb_pitch = 0, wzf_pitch = 0;
  uint16_t* wZb = nullptr;           // [wcap x wzb_pitch] bf16 (full mean or SNP partial)
  float* wZf = nullptr;              // [wcap x wzf_pitch] fp32 mode
  uint16_t* wGb = nullptr;           // [wcap x gb_pitch] gathered dL/dpre (bf16 mode)
  float* wGf = nullptr;              // [wcap x h_pitch] (fp32 mode)
  // NFP: the rank's column slice [col_lo, col_hi) of W^1 (column-owned, no all-reduce)
  int col_lo = 0, col_hi = 0;
  int64_t ws_pitch = 0;
  float* W1s = nullptr;              // [d_out x w_cols]
  uint16_t* Wb1s = nullptr;          // [d_out x ws_pitch]
  float* dW1s = nullptr;             // [d_out x w_cols]
};

// GAT first layer (gat.cu).  Every strategy runs as owners
// processing work items (GDP: the rank's own rows); per item the owner keeps the
// per-head aggregate Z^h = sum_u alpha_vu^h x_u, the LeakyReLU scores and the
// softmax statistics for the backward.
struct GatState {
  int H = 0, F = 0;                  // heads, per-head width (d_out = H*F)
  int cols = 0;                      // aggregated feature columns (d, or the NFP slice)
  int64_t zp = 0;                    // per-head pitch of Z (elements); an item's Z row is H*zp
  int64_t icap = 0;                  // item capacity
  float* a_src = nullptr;            // [d_out] attention vectors (replicated)
  float* a_dst = nullptr;
  float* da_src = nullptr;           // [d_out] in the flat gradient buffer (after db^1)
  float* da_dst = nullptr;
  float* wt = nullptr;               // [2][H][cols] w~ = W^hT a^h (src, dst)
  float* dwt = nullptr;              // [2][H][cols] dL/dw~ accumulators
  void* Z = nullptr;                 // [icap][H][zp] bf16 or fp32
  float* esc = nullptr;              // [icap*k][H] LeakyReLU scores
  float* Lm = nullptr;               // [icap][H] log-sum-exp (SNP: the partial max m_c)
  float* Ss = nullptr;               // [icap][H] SNP: partial sum S_c
  float* Lb = nullptr;               // [icap][H] backward: the (global) log-sum-exp of the item
  float* tb = nullptr;               // [icap][H] backward: t = g . (pre - b) of the item
  float* wG = nullptr;               // [icap][d_out] gathered g (fp32)
  float* wGs = nullptr;              // [icap][d_out] g scaled by the SNP merge weight (else == wG)
  uint16_t* wGb = nullptr;           // bf16 mode: [icap][wpb] gathered g (tcgen05 operands; tail rows zero)
  uint16_t* wGsb = nullptr;          // bf16 mode: ... scaled by the SNP merge weight (else == wGb)
  int64_t wpb = 0;
  float* Gam = nullptr;              // [icap][H][gp] gamma^h = W^hT g^h
  int64_t gp = 0;                    // per-head pitch of Gam (floats, multiple of 4)
  float** otab = nullptr;            // [H][C] routed projection targets per head
  // requester side
  float* t = nullptr;                // [max_rows][H]
  float* Lr = nullptr;               // [max_rows][H] SNP: merged log-sum-exp
  float* slot = nullptr;             // SNP: [max_rows][C][slot_pitch] partial (Q, m_c, S_c)
  int64_t slot_pitch = 0;
  float* ssum = nullptr;             // NFP: [max_rows][k][H] summed partial scores
  float* dsum = nullptr;             // NFP: [max_rows][k][H] summed partial dalpha
};

// The sampled mini-batch of one step (seeds, K hops, block transposes).  Two per
// rank: step t+1 is sampled into one while step t computes on the other.
struct SampleSet {
  uint16_t* z1b = nullptr;          // layer-1 Z of this batch (bf16 / fp32 mode): with the pipeline the
  float* z1f = nullptr;             //   sampling branch also aggregates it (z_prefetch)
  int32_t* seeds = nullptr;
  int32_t* small = nullptr;         // [0] n_seeds [1] n_global
  uint64_t* step_cell = nullptr;    // step id of the batch held here (Philox key of its samples)
  std::vector<Hop> hops;
};

struct RankState {
  int rank = 0;
  SampleSet sset[2];
  // the set the current step computes on (copies of sset[active]'s fields)
  int32_t* seeds = nullptr;
  int32_t* small = nullptr;
  std::vector<Hop> hops;
  std::vector<Layer> L;
  uint32_t* dst_bm = nullptr;
  uint32_t* new_bm = nullptr;
  int32_t* pos = nullptr;
  int32_t* partials = nullptr;
  float* loss = nullptr;
  int32_t* ce_ws = nullptr;          // ce_loss: block-partial losses + ticket (zeroed once, self-resetting)
  Xchg x;
  GatState ga;
};

}  // namespace apt

struct apt_trainer {
  apt_ctx* ctx = nullptr;
  const apt_graph* g = nullptr;
  const apt_fstore* f = nullptr;
  apt_model_desc m{};
  apt_strategy s = APT_GDP;
  int K = 0, world = 1;
  int32_t* labels = nullptr;
  int32_t* perm = nullptr;
  int64_t n_train = 0, steps_per_epoch = 1;
  uint64_t* step_cells = nullptr;    // [2] step id of the batch in sample set 0 / 1
  uint64_t* step_dev = nullptr;      // step cell of the set being computed (sset[parity].step_cell)
  std::vector<apt::RankState> R;
  // device pointer tables for cross-rank kernels (peer pointers in a multi-GPU job)
  float** dW_tab = nullptr;
  float** H1_tab = nullptr;          // requesters' layer-1 outputs
  std::vector<float*> h1_host;       // ... the same pointers on the host
  float** G1_tab = nullptr;          // requesters' layer-1 dL/dpre (fp32)
  uint16_t** Gb1_tab = nullptr;      // ... bf16
  int32_t** wn_tab = nullptr;        // owners' work counters / lists
  int32_t** wrank_tab = nullptr;
  int32_t** wrow_tab = nullptr;
  int32_t** wgid_tab = nullptr;
  // GAT first layer (gat_heads > 0): requesters' buffers seen by every rank
  int gat_heads = 0;
  float** gt_tab = nullptr;          // t
  float** gL_tab = nullptr;          // SNP merged log-sum-exp
  float** slot_tab = nullptr;        // SNP partial slots
  float** ssum_tab = nullptr;        // NFP score sums
  float** dsum_tab = nullptr;        // NFP dalpha sums
  float** gG_tab = nullptr;          // requesters' G (fp32)
  uint16_t** gGb_tab = nullptr;      // requesters' Gb (bf16)
  bool use_graph = false;
  bool capturing = false;
  bool tapped = false;
  bool pfork_recorded = false;       // fork point 3: the sampling branch's fork event was recorded at the step start               // a captured timing event hangs off the chain on ctx->tap (join before EndCapture)
  // pipelining: step t+1 is sampled on ctx->samp while step t computes
  bool pipeline = true;
  bool z_prefetch = false;           // GDP SAGE layer 1: the next batch's gather+mean runs on the sampling
                                     //   branch (it reads only the static features), beside this step
  bool z_ready = false;              // the active set's layer-1 Z is already aggregated
  int z_where = 1;                   // z_prefetch: 1 on the sampling branch, 2 beside this step's backward tail
  int z_next = -1;                   // z_where 2: the set whose Z this step aggregates (pipelined bodies)
  cudaEvent_t ev_zt = nullptr, ev_zf = nullptr;   // tail prefetch: fork point / done
  int parity = 0;                    // sample set the last step computed on
  int64_t primed = -1;               // step id already sampled into sset[primed_parity]
  int primed_parity = 0;
  bool csc_forked = false;
  bool out_dz_fused = false;    // the fused output-layer kernel also wrote dZ^K (bf16 / deg)
  bool bg_csc_forked = false;   // the background sampling forked its transposes onto ctx->samp2
  std::function<apt_status()> deferred_fork;   // pipelined: next-step sampling, launched after the layer-1 forward
  cudaGraphExec_t gexec_p[2][2] = {};   // [parity][update] pipelined step graphs
  cudaGraph_t graph_p[2][2] = {};
  cudaGraphNode_t step_node_p[2][2] = {};
  int64_t launches_p[2][2] = {};
  cudaGraphExec_t gexec = nullptr;
  cudaGraphExec_t gexec_host = nullptr;   // the end-to-end step: H2D batch, step, D2H loss
  cudaGraph_t graph_host = nullptr;
  cudaGraphNode_t step_node_host = nullptr;
  int graph_host_update = -1;
  int64_t launches_per_step_host = 0;
  int32_t* hb_pinned = nullptr;       // [2][1 + C*B] host staging per sample set: n, ids (pinned)
  int32_t* hb_dev = nullptr;          // [2][1 + C*B] device copies
  int64_t hb_len = 0;                 // 1 + C*B
  // pipelined end-to-end calls: batch submitted by the previous call, sampled into set
  bool host_primed = false;
  int host_parity = 0;
  cudaGraphExec_t gexec_hp[2][2] = {};
  cudaGraph_t graph_hp[2][2] = {};
  cudaGraphNode_t step_node_hp[2][2] = {};
  int64_t launches_hp[2][2] = {};
  float* loss_pinned = nullptr;       // [2][APT_MAX_RANKS] per sample-set parity, per hosted rank
  cudaEvent_t ev_done[2] = {};        // end of the step graph of each parity (async end-to-end calls)
  bool async_pending = false;         // an async call launched a step whose loss is not yet returned
  cudaGraph_t graph = nullptr;
  cudaGraphNode_t step_node = nullptr;
  int64_t launches_per_step = 0;
  float* ar_scratch = nullptr;       // multi-process all-reduce: sum of the peers' gradients
  std::vector<void*> peer_opened;    // IPC mappings of peer buffers
  int graph_update = -1;
  cudaEvent_t ev[8] = {};
  bool ev_ok = false;
  double last_agg_bytes = 0;
  apt::Arena arena;
  ~apt_trainer() { apt::close_peers(peer_opened); apt::defer_exported(ctx, arena); }
};

namespace apt {
// A timing event at the current point of stream st.  Eagerly: a plain record.  Inside a
// stream capture the record node hangs off the chain on ctx->tap (an internal fork edge),
// so the kernel that follows on st keeps its programmatic (PDL) edge to the one before:
// an external record node placed IN the chain cost the step ~5 us per event (measured
// with tools/timeline.py: the next kernel waited for the full drain + the node).
// APT_TAP_EVENTS=0 puts them back in the chain (A/B).
inline cudaError_t tap_event(apt_trainer* t, cudaEvent_t ev, cudaStream_t st, bool in_chain = false) {
  static const int tap = [] { const char* v = std::getenv("APT_TAP_EVENTS"); return v ? atoi(v) : 1; }();
  if (!t->capturing) return cudaEventRecord(ev, st);
  if (!tap || in_chain) return cudaEventRecordWithFlags(ev, st, cudaEventRecordExternal);
  apt_ctx* c = t->ctx;
  cudaError_t e = cudaEventRecord(c->ev_tap, st);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(c->tap, c->ev_tap, 0);
  if (e == cudaSuccess) e = cudaEventRecordWithFlags(ev, c->tap, cudaEventRecordExternal);
  t->tapped = true;
  return e;
}
// Join the tap branch into the capture origin (every forked stream must rejoin before
// cudaStreamEndCapture); call right before it.
inline cudaError_t tap_join(apt_trainer* t) {
  if (!t->tapped) return cudaSuccess;
  t->tapped = false;
  apt_ctx* c = t->ctx;
  cudaError_t e = cudaEventRecord(c->ev_tapj, c->tap);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(c->stream, c->ev_tapj, 0);
  return e;
}
}  // namespace apt
