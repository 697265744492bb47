// dryrun.cu -- APT's Planner inputs: the dry-run counters and
// the bandwidth trials of the exchange operators.
//
// Dry-run (reading Z13): for `n_steps` steps of the current epoch and every
// strategy, sample every rank's mini-batch exactly as the trainer would (seeds by
// chunk for GDP/NFP, by partition for SNP/DNP), then count -- without
// loading features or training -- what Permute/Shuffle/Execute/Reshuffle
// would move for the first layer: layer-1 destinations N_d, virtual nodes N_vs /
// N_vd, unique feature rows per tier (local HBM / NVLink peer),
// computation-graph bytes and hidden-embedding bytes of each message (the message
// formats of DESIGN.md §Messages, oracle/strategy.py).  Sampling is a pure
// function of (seed, node, hop, step) (reading Z2), so every process of a job can
// count every rank's blocks without communication.  T_build is measured:
// the device time of each rank's sampling.
//
// Counting is set-based: "unique rows read by owner c" is a bitmap per owner,
// test-and-set with atomicOr, counted the moment a bit flips.
#include <algorithm>
#include <chrono>
#include <cstring>
#include <vector>

#include "common.cuh"
#include "trainer.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what);
}  // namespace apt

#define CK(ctx, expr)                                        \
  do {                                                       \
    apt_status _s = ::apt::check_cuda((ctx), (expr), #expr); \
    if (_s != APT_OK) return _s;                             \
  } while (0)

namespace apt {

// Per (strategy, requester) device counters.  pair_* are per step (folded into
// the totals and cleared by fold_kernel); C <= 8.
struct DryCounters {
  unsigned long long n_d[APT_MAX_RANKS];
  unsigned long long edges[APT_MAX_RANKS];                    // layer-1 sampled edges of block r
  unsigned long long uniq[APT_MAX_RANKS];                     // GDP/NFP: unique sources of block r
  unsigned long long rows_local[APT_MAX_RANKS];               // per owner
  unsigned long long rows_peer[APT_MAX_RANKS];
  unsigned long long rows_host[APT_MAX_RANKS];
  unsigned long long pair_rows[APT_MAX_RANKS][APT_MAX_RANKS]; // this step: rows of requester r sent to owner c
  unsigned long long pair_edges[APT_MAX_RANKS][APT_MAX_RANKS];
  unsigned long long tot_rows[APT_MAX_RANKS][APT_MAX_RANKS];
  unsigned long long tot_edges[APT_MAX_RANKS][APT_MAX_RANKS];
  unsigned long long tot_msgs[APT_MAX_RANKS][APT_MAX_RANKS];  // steps in which the (r, c) message was non-empty
};

// Where rank r reads node u from (the unified store's tiers): 0 local HBM (own shard or
// own cache), 1 NVLink peer, 2 host tier.
struct TierInfo {
  const int32_t* part; const int32_t* lrow; const int64_t* rows; const uint32_t* cache_bm; int64_t n_words;
  const uint32_t* any_bm;   // P:163 caches: cached by some GPU (else the row is on the host only)
  __device__ __forceinline__ int of(int u, int r) const {
    if (cache_bm && (cache_bm[int64_t(r) * n_words + (u >> 5)] >> (u & 31) & 1u)) return 0;
    if (any_bm) return (any_bm[u >> 5] >> (u & 31) & 1u) ? 1 : 2;
    const int o = part[u];
    if (rows && lrow[u] >= rows[o]) return 2;
    return o == r ? 0 : 1;
  }
};

__device__ __forceinline__ bool test_and_set(uint32_t* bm, int u) {
  const uint32_t bit = 1u << (u & 31);
  return (atomicOr(bm + (u >> 5), bit) & bit) == 0;
}

// One thread per layer-1 row of requester r (ELL cnt/nbr of the layer-1 hop).
__global__ void dry_count_kernel(int S, int r, int C, const int32_t* __restrict__ dst, const int32_t* __restrict__ n_p,
                                 const int32_t* __restrict__ cnt, const int32_t* __restrict__ nbr, int k,
                                 const int32_t* __restrict__ part, uint32_t* bm, int64_t n_words, DryCounters* dc,
                                 TierInfo ti) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int v = dst[i];
    const int c_i = cnt[i];
    const int32_t* row = nbr + i * k;
    atomicAdd(&dc->edges[r], (unsigned long long)c_i);
    if (S == APT_GDP || S == APT_NFP) {
      uint32_t* b = bm + int64_t(r) * n_words;      // unique sources of block r
      for (int e = 0; e < c_i; ++e) {
        const int u = row[e];
        if (test_and_set(b, u)) {
          atomicAdd(&dc->uniq[r], 1ull);
          if (S == APT_GDP) {
            const int tr = ti.of(u, r);
            atomicAdd(tr == 0 ? &dc->rows_local[r] : tr == 1 ? &dc->rows_peer[r] : &dc->rows_host[r], 1ull);
          }
        }
      }
    } else if (S == APT_SNP) {
      int ec[APT_MAX_RANKS];
#pragma unroll
      for (int c = 0; c < APT_MAX_RANKS; ++c) ec[c] = 0;
      for (int e = 0; e < c_i; ++e) {
        const int u = row[e];
        const int c = part[u];
        ++ec[c];
        if (test_and_set(bm + int64_t(c) * n_words, u))   // SNP reads its own partition: HBM or host tier
          atomicAdd(ti.of(u, c) == 2 ? &dc->rows_host[c] : &dc->rows_local[c], 1ull);
      }
#pragma unroll
      for (int c = 0; c < APT_MAX_RANKS; ++c)
        if (c < C && ec[c]) {
          atomicAdd(&dc->pair_rows[r][c], 1ull);
          atomicAdd(&dc->pair_edges[r][c], (unsigned long long)ec[c]);
        }
    } else {   // DNP: the row goes to its owner, which reads all of its sources
      const int o = part[v];
      atomicAdd(&dc->pair_rows[r][o], 1ull);
      atomicAdd(&dc->pair_edges[r][o], (unsigned long long)c_i);
      for (int e = 0; e < c_i; ++e) {
        const int u = row[e];
        if (test_and_set(bm + int64_t(o) * n_words, u)) {
          const int to = ti.of(u, o);
          atomicAdd(to == 0 ? &dc->rows_local[o] : to == 1 ? &dc->rows_peer[o] : &dc->rows_host[o], 1ull);
        }
      }
    }
  }
}

__global__ void dry_nd_kernel(int r, const int32_t* __restrict__ n_p, DryCounters* dc) {
  APT_PDL_PROLOGUE();
  if (threadIdx.x == 0) dc->n_d[r] += *n_p;
}

__global__ void dry_fold_kernel(int C, DryCounters* dc) {
  APT_PDL_PROLOGUE();
  const int t = threadIdx.x;
  if (t < C * C) {
    const int r = t / C, c = t % C;
    const unsigned long long rows = dc->pair_rows[r][c];
    dc->tot_rows[r][c] += rows;
    dc->tot_edges[r][c] += dc->pair_edges[r][c];
    dc->tot_msgs[r][c] += rows > 0 ? 1 : 0;
    dc->pair_rows[r][c] = 0;
    dc->pair_edges[r][c] = 0;
  }
}

__global__ void dry_set_step_kernel(uint64_t* p, uint64_t v) {
  APT_PDL_PROLOGUE(); *p = v; }

}  // namespace apt

using namespace apt;

namespace {
// The dry run's sampler: seed selection + K hops of sampling/compaction for one
// (rank, step) of the current epoch into its own buffers (no feature loading, no
// training).  Shared by apt_dryrun and apt_access_counts.
struct DrySampler {
  apt_trainer* t;
  Arena A;
  int64_t n_words = 0;
  int32_t *seeds = nullptr, *small = nullptr, *pos = nullptr, *partials = nullptr;
  uint32_t *dst_bm = nullptr, *new_bm = nullptr;
  uint64_t* step_dev = nullptr;
  std::vector<Hop> hops;
  bool init(apt_trainer* tr) {
    t = tr;
    const int C = t->world, K = t->K;
    const apt_graph* g = t->g;
    n_words = ceil_div(g->n, 32);
    // sampler state sized for the largest seed set (SNP/DNP: up to C*B on one rank)
    const int64_t B0 = int64_t(C) * t->m.batch;
    seeds = A.alloc<int32_t>(B0, false);
    small = A.alloc<int32_t>(16, true);
    dst_bm = A.alloc<uint32_t>(n_words, true);
    new_bm = A.alloc<uint32_t>(n_words, true);
    pos = A.alloc<int32_t>(g->n, false);
    partials = A.alloc<int32_t>(2 * ceil_div(n_words, kScanWsTile) + 8, false);
    step_dev = A.alloc<uint64_t>(1, true);
    hops.resize(K);
    int64_t maxF = B0;
    const int32_t* dst = seeds;
    const int32_t* n_dst = small;
    for (int h = 0; h < K; ++h) {
      Hop& hp = hops[h];
      hp.k = t->m.fanouts[K - 1 - h];
      hp.max_dst = maxF;
      hp.max_src = std::max<int64_t>(maxF, std::min<int64_t>(maxF * (1 + hp.k), g->n));
      hp.dst = dst;
      hp.n_dst = n_dst;
      hp.cnt = A.alloc<int32_t>(maxF, true);
      hp.nbr = A.alloc<int32_t>(maxF * hp.k, false);
      hp.counts = A.alloc<int32_t>(4, true);
      hp.part2 = A.alloc<int32_t>(2 * ceil_div(maxF, kScanWsTile) + 8, false);
      if (h + 1 < K) {
        hp.src = A.alloc<int32_t>(hp.max_src, false);
        hp.indptr = A.alloc<int32_t>(maxF + 1, true);
        hp.indices = A.alloc<int32_t>(maxF * hp.k, false);
      }
      dst = hp.src;
      n_dst = hp.counts;
      maxF = hp.max_src;
    }
    return seeds && step_dev && hops[K - 1].nbr && (K == 1 || hops[K - 2].indices);
  }
  void set_step(int64_t st, cudaStream_t s) { dry_set_step_kernel<<<1, 1, 0, s>>>(step_dev, uint64_t(st)); }
  // rank r's seeds of the current step (by_part: its partition's seeds, SNP/DNP) and its blocks
  // e0 / e1 (optional): recorded around the layer-1 hop's sampling
  apt_status sample(int r, bool by_part, cudaEvent_t e0 = nullptr, cudaEvent_t e1 = nullptr) {
    apt_ctx* c = t->ctx;
    const int C = t->world, K = t->K;
    const apt_graph* g = t->g;
    SeedArgs sa{t->perm, t->n_train, step_dev, t->steps_per_epoch, C, r, t->m.batch, by_part ? 1 : 0, g->part,
                seeds, small, small + 1};
    CK(c, launch_select_seeds(sa, c->stream));
    for (int h = 0; h < K; ++h) {
      Hop& hp = hops[h];
      SampleArgs sm{g->indptr, g->indices, hp.dst, hp.n_dst, hp.max_dst, hp.k,
                    philox_key(t->m.sample_seed, kDomSample), step_dev, h, hp.cnt, hp.nbr};
      if (h == K - 1 && e0) CK(c, cudaEventRecord(e0, c->stream));
      CK(c, launch_sample(sm, c->stream));
      if (h == K - 1 && e1) CK(c, cudaEventRecord(e1, c->stream));
      if (h + 1 < K) {
        CompactArgs ca{hp.dst, hp.n_dst, hp.max_dst, hp.cnt, hp.nbr, hp.k, dst_bm, new_bm, n_words, pos, hp.src,
                       hp.counts, hp.indptr, hp.indices, hp.counts + 1, partials, hp.part2};
        CK(c, launch_compact(ca, c->stream));
      }
    }
    c->launches += 1 + 4 * K;
    return APT_OK;
  }
};
}  // namespace

extern "C" apt_status apt_dryrun(apt_trainer* t, int64_t n_steps, apt_plan_stats* out) {
  if (!t || !out || n_steps < 1) return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "apt_dryrun: bad arguments");
  if (!t->perm) return set_err(t->ctx, APT_E_STATE, "apt_dryrun: call apt_trainer_set_epoch first");
  apt_ctx* c = t->ctx;
  const int C = t->world, K = t->K;
  const apt_graph* g = t->g;
  n_steps = std::min<int64_t>(n_steps, t->steps_per_epoch);
  DrySampler ds;
  const bool ok = ds.init(t);
  Arena& A = ds.A;
  const int64_t n_words = ds.n_words;
  uint32_t* own_bm = A.alloc<uint32_t>(n_words * C, true);        // one bitmap per owner / block
  DryCounters* dc = A.alloc<DryCounters>(4, true);                 // per strategy
  std::vector<Hop>& hops = ds.hops;
  if (!ok || !own_bm || !dc) return set_err(c, APT_E_OOM, "apt_dryrun: out of device memory");
  // tiers of the unified store (rows beyond the HBM budgets, replicated hot rows)
  const TierInfo ti{g->part, g->lrow, t->f->tiered ? t->f->rows_dev : nullptr, t->f->cache_bm, n_words,
                    t->f->p163 ? t->f->any_bm : nullptr};
  std::vector<cudaEvent_t> ev, ev1;   // per (strategy, step, rank): whole sampling / the layer-1 hop
  struct Mark { int s, r; };
  std::vector<Mark> marks;
  const auto wall0 = std::chrono::steady_clock::now();
  auto new_event = [&]() {
    cudaEvent_t e;
    cudaEventCreate(&e);
    ev.push_back(e);
    return e;
  };
  for (int S = 0; S < 4; ++S) {
    const bool by_part = (S == APT_SNP || S == APT_DNP) && C > 1;
    for (int64_t st = 0; st < n_steps; ++st) {
      ds.set_step(st, c->stream);
      CK(c, cudaMemsetAsync(own_bm, 0, sizeof(uint32_t) * n_words * C, c->stream));
      for (int r = 0; r < C; ++r) {
        CK(c, cudaEventRecord(new_event(), c->stream));
        cudaEvent_t h0, h1;
        cudaEventCreate(&h0);
        cudaEventCreate(&h1);
        ev1.push_back(h0);
        ev1.push_back(h1);
        { apt_status s2 = ds.sample(r, by_part, h0, h1); if (s2 != APT_OK) return s2; }
        CK(c, cudaEventRecord(new_event(), c->stream));
        marks.push_back({S, r});
        const Hop& l1 = hops[K - 1];
        launch_pdl(dry_nd_kernel, dim3(1), dim3(32), 0, c->stream, r, l1.n_dst, dc + S);
        const int64_t blocks = grid_cap(ceil_div(l1.max_dst, 256), 8);
        launch_pdl(dry_count_kernel, dim3(blocks), dim3(256), 0, c->stream, S, r, C, l1.dst, l1.n_dst, l1.cnt, l1.nbr, l1.k, g->part,
                                                        own_bm, n_words, dc + S, ti);
        CK(c, cudaGetLastError());
        c->launches += 3;
      }
      launch_pdl(dry_fold_kernel, dim3(1), dim3(64), 0, c->stream, C, dc + S);
      CK(c, cudaGetLastError());
    }
  }
  CK(c, cudaStreamSynchronize(c->stream));
  DryCounters h[4];
  CK(c, cudaMemcpy(h, dc, sizeof h, cudaMemcpyDeviceToHost));
  // T_build per (strategy, rank): device time of the rank's seed selection + sampling
  double tb[4][APT_MAX_RANKS] = {};
  double t_l1 = 0.0;   // layer-1 hop sampling, summed over every (strategy, step, rank)
  for (size_t i = 0; i < marks.size(); ++i) {
    float ms = 0.f, ms1 = 0.f;
    cudaEventElapsedTime(&ms, ev[2 * i], ev[2 * i + 1]);
    cudaEventElapsedTime(&ms1, ev1[2 * i], ev1[2 * i + 1]);
    tb[marks[i].s][marks[i].r] += ms * 1e-3;
    t_l1 += ms1 * 1e-3;
  }
  for (auto e : ev) cudaEventDestroy(e);
  for (auto e : ev1) cudaEventDestroy(e);
  unsigned long long rows_l1 = 0;
  for (int S = 0; S < 4; ++S)
    for (int r = 0; r < C; ++r) rows_l1 += h[S].n_d[r];
  // reading R1: an owner RE-SAMPLES the layer-1 rows other requesters send it (NFP: every
  // other block; SNP / DNP: the items routed to it), at the measured layer-1 sampling
  // cost per row -- part of its T_build ("sending part of their computation graphs")
  const double per_row = rows_l1 ? t_l1 / double(rows_l1) : 0.0;
  double tr[4][APT_MAX_RANKS] = {};
  for (int cc = 0; cc < C && C > 1; ++cc) {
    for (int b = 0; b < C; ++b)
      if (b != cc) {
        tr[APT_NFP][cc] += per_row * double(h[APT_NFP].n_d[b]);
        tr[APT_SNP][cc] += per_row * double(h[APT_SNP].tot_rows[b][cc]);
        tr[APT_DNP][cc] += per_row * double(h[APT_DNP].tot_rows[b][cc]);
      }
  }

  // ---- assemble the Planner statistics (message formats: oracle/strategy.py)
  memset(out, 0, sizeof *out);
  out->world = C;
  out->steps = n_steps;
  const int64_t d = g ? t->m.dims[0] : 0, dd = t->m.dims[1];
  const int64_t bf = t->m.dtype == APT_BF16 ? 2 : 4, bh = 4;
  const int64_t calls = C > 1 ? 3 * n_steps : 0;
  for (int S = 0; S < 4; ++S)
    for (int r = 0; r < C; ++r) {
      out->n_d[S][r] = h[S].n_d[r];
      out->t_resample_s[S][r] = tr[S][r];
      out->t_build_s[S][r] = tb[S][r] + tr[S][r];
    }
  // GDP: local / peer / host rows of each requester's own block
  for (int r = 0; r < C; ++r) {
    out->rows_local[APT_GDP][r] = h[APT_GDP].rows_local[r];
    out->rows_peer[APT_GDP][r] = h[APT_GDP].rows_peer[r];
    out->rows_host[APT_GDP][r] = h[APT_GDP].rows_host[r];
  }
  // NFP: every rank reads the unique sources of every block, its column slice only;
  // receives every other block (AllBroadcast), sends (C-1) partials per own row
  {
    const DryCounters& q = h[APT_NFP];
    unsigned long long all_uniq = 0;
    for (int b = 0; b < C; ++b) all_uniq += q.uniq[b];
    for (int cc = 0; cc < C; ++cc) {
      out->rows_local[APT_NFP][cc] = all_uniq;
      const int64_t lo = (int64_t(cc) * d) / C, hi = (int64_t(cc + 1) * d) / C;
      out->feat_bytes_local[APT_NFP][cc] = all_uniq * (hi - lo) * bf;
      for (int b = 0; b < C; ++b)
        if (b != cc) {
          out->graph_bytes[APT_NFP][cc] += 4 * (3 * n_steps + 3 * q.n_d[b] + q.edges[b]);
          out->hidden_bytes_bwd[APT_NFP][cc] += q.n_d[b] * dd * bh;
        }
      out->hidden_bytes_fwd[APT_NFP][cc] = int64_t(C - 1) * q.n_d[cc] * dd * bh;
      out->n_calls[APT_NFP][cc] = calls;
    }
  }
  // SNP: virtual nodes (r -> c != r), local reads only
  {
    const DryCounters& q = h[APT_SNP];
    for (int cc = 0; cc < C; ++cc) {
      out->rows_local[APT_SNP][cc] = q.rows_local[cc];
      out->rows_host[APT_SNP][cc] = q.rows_host[cc];
    }
    for (int r = 0; r < C; ++r)
      for (int cc = 0; cc < C; ++cc) {
        if (r == cc) continue;
        out->n_vs[r] += q.tot_rows[r][cc];
        out->graph_bytes[APT_SNP][cc] += 4 * (3 * q.tot_msgs[r][cc] + 3 * q.tot_rows[r][cc] + q.tot_edges[r][cc]);
        out->hidden_bytes_fwd[APT_SNP][r] += q.tot_rows[r][cc] * dd * bh;
        out->hidden_bytes_bwd[APT_SNP][cc] += q.tot_rows[r][cc] * dd * bh;
      }
    for (int r = 0; r < C; ++r) out->n_calls[APT_SNP][r] = calls;
  }
  // DNP: rows shipped to their owner (ids only), owners read local + halo rows
  {
    const DryCounters& q = h[APT_DNP];
    for (int o = 0; o < C; ++o) {
      out->rows_local[APT_DNP][o] = q.rows_local[o];
      out->rows_peer[APT_DNP][o] = q.rows_peer[o];
      out->rows_host[APT_DNP][o] = q.rows_host[o];
    }
    for (int r = 0; r < C; ++r)
      for (int o = 0; o < C; ++o) {
        if (r == o) continue;
        out->n_vd[r] += q.tot_rows[r][o];
        out->graph_bytes[APT_DNP][o] += 4 * (2 * q.tot_msgs[r][o] + 2 * q.tot_rows[r][o]);
        out->hidden_bytes_fwd[APT_DNP][r] += q.tot_rows[r][o] * dd * bh;
        out->hidden_bytes_bwd[APT_DNP][o] += q.tot_rows[r][o] * dd * bh;
      }
    for (int r = 0; r < C; ++r) out->n_calls[APT_DNP][r] = calls;
  }
  for (int S = 0; S < 4; ++S)
    for (int r = 0; r < C; ++r) {
      if (S != APT_NFP) out->feat_bytes_local[S][r] = out->rows_local[S][r] * d * bf;
      out->feat_bytes_peer[S][r] = out->rows_peer[S][r] * d * bf;
      out->feat_bytes_host[S][r] = out->rows_host[S][r] * d * bf;
    }
  // GAT layer 1: attention's extra exchanges (apt.h; oracle/strategy.py emulate_layer1)
  const int64_t H = t->gat_heads;
  out->gat_heads = int(H);
  if (H > 0 && C > 1) {
    const DryCounters& qn = h[APT_NFP];
    for (int cc = 0; cc < C; ++cc)
      for (int b = 0; b < C; ++b)
        if (b != cc) out->attn_bytes[APT_NFP][cc] += 4 * H * 4 * int64_t(qn.edges[b]);
    const DryCounters& qs = h[APT_SNP];
    for (int r = 0; r < C; ++r)
      for (int cc = 0; cc < C; ++cc) {
        out->attn_feat_bytes[APT_SNP][cc] += int64_t(qs.tot_rows[r][cc]) * d * bf;
        if (r == cc) continue;
        out->attn_bytes[APT_SNP][r] += int64_t(qs.tot_rows[r][cc]) * 2 * H * 4;
        out->attn_bytes[APT_SNP][cc] += int64_t(qs.tot_rows[r][cc]) * 2 * H * 4;
      }
  }
  out->t_dryrun_s = std::chrono::duration<double>(std::chrono::steady_clock::now() - wall0).count();
  return APT_OK;
}

// ---------------------------------------------------------------- access frequencies
// How often each node's input row is loaded (Table 3, "Node access
// skewness"; reading R12): once per (step, requester) in which it is a source of the
// requester's layer-1 block, over the first n_steps global steps of the epoch under
// GDP's seed split.  Drives the excess cache's hot list.
namespace apt {
__global__ void access_count_kernel(const int32_t* __restrict__ n_p, const int32_t* __restrict__ cnt,
                                    const int32_t* __restrict__ nbr, int k, uint32_t* bm, int32_t* counts) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int c_i = cnt[i];
    for (int e = 0; e < c_i; ++e) {
      const int u = nbr[i * k + e];
      if (test_and_set(bm, u)) atomicAdd(counts + u, 1);
    }
  }
}
}  // namespace apt

extern "C" apt_status apt_access_counts(apt_trainer* t, int64_t n_steps, int32_t* counts_host) {
  if (!t || !counts_host || n_steps < 1)
    return set_err(t ? t->ctx : nullptr, APT_E_INVALID, "apt_access_counts: bad arguments");
  if (!t->perm) return set_err(t->ctx, APT_E_STATE, "apt_access_counts: call apt_trainer_set_epoch first");
  apt_ctx* c = t->ctx;
  const int C = t->world, K = t->K;
  n_steps = std::min<int64_t>(n_steps, t->steps_per_epoch);
  DrySampler ds;
  const bool ok = ds.init(t);
  uint32_t* bm = ds.A.alloc<uint32_t>(ds.n_words, true);
  int32_t* counts = ds.A.alloc<int32_t>(t->g->n, true);
  if (!ok || !bm || !counts) return set_err(c, APT_E_OOM, "apt_access_counts: out of device memory");
  const Hop& l1 = ds.hops[K - 1];
  const int64_t blocks = grid_cap(ceil_div(l1.max_dst, 256), 8);
  for (int64_t st = 0; st < n_steps; ++st) {
    ds.set_step(st, c->stream);
    for (int r = 0; r < C; ++r) {
      CK(c, cudaMemsetAsync(bm, 0, sizeof(uint32_t) * ds.n_words, c->stream));
      { apt_status s = ds.sample(r, false); if (s != APT_OK) return s; }
      launch_pdl(access_count_kernel, dim3(blocks), dim3(256), 0, c->stream, l1.n_dst, l1.cnt, l1.nbr, l1.k, bm, counts);
      CK(c, cudaGetLastError());
      c->launches++;
    }
  }
  CK(c, cudaMemcpyAsync(counts_host, counts, sizeof(int32_t) * t->g->n, cudaMemcpyDeviceToHost, c->stream));
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

// Hot list for the excess cache: node ids by descending access count, ties by
// ascending id (host arithmetic).
extern "C" apt_status apt_hot_rows(const int32_t* counts, int64_t n, int64_t k, int64_t* ids_out) {
  if (!counts || !ids_out || n < 0 || k < 0 || k > n) return APT_E_INVALID;
  std::vector<int64_t> idx(static_cast<size_t>(n));
  for (int64_t i = 0; i < n; ++i) idx[size_t(i)] = i;
  std::partial_sort(idx.begin(), idx.begin() + k, idx.end(), [&](int64_t a, int64_t b) {
    return counts[a] != counts[b] ? counts[a] > counts[b] : a < b;
  });
  std::copy(idx.begin(), idx.begin() + k, ids_out);
  return APT_OK;
}

// ---------------------------------------------------------------- link trials
// Bandwidth trials ("measures the bandwidth of different communication
// operators").  Each operator is timed at two message sizes (CUDA events,
// best of 5) and fitted to t = alpha + bytes / beta.  Operators this process can
// run are measured: the local HBM row gather (the unified store's local tier) and
// a device-to-device copy; peer operators need a second GPU -- with one device
// (world 1 or the emulated job) they take the measured NVLink references of this
// pool (peer copy 770 GB/s per direction, 8-rank all-reduce bus 725 GB/s; per-call
// latency of a fused peer-memory exchange ~ 3 us) and `measured` says which.
namespace apt {
__global__ void trial_gather_kernel(const uint4* __restrict__ src, int64_t n_rows, int vec_per_row,
                                    const int32_t* __restrict__ ids, int64_t n, uint4* __restrict__ out) {
  const int64_t total = n * vec_per_row;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = t / vec_per_row;
    const int j = int(t - i * vec_per_row);
    out[t] = ld_nc_v4(src + int64_t(ids[i]) * vec_per_row + j);
  }
}
__global__ void trial_ids_kernel(int32_t* ids, int64_t n, int64_t n_rows, uint32_t salt) {
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < n; t += int64_t(gridDim.x) * blockDim.x) {
    uint32_t h = uint32_t(t) * 2654435761u ^ salt;
    h ^= h >> 16; h *= 0x7feb352du; h ^= h >> 15;
    ids[t] = int32_t(h % uint32_t(n_rows));
  }
}
// Peer-operator trials (one process per GPU): the same row gather reading another
// rank's table (pull), writing into it (push), rows spread over every peer
// (all-to-all), whole chunks from every peer (all-gather), chunk sums over the peers
// (reduce-scatter: the fused Reshuffle's reduce) and full sums (all-reduce).
__global__ void trial_peer_gather_kernel(const uint4* const* __restrict__ tab, int C, int self, int mode,
                                         int64_t n_rows, int vec_per_row, const int32_t* __restrict__ ids, int64_t n,
                                         uint4* __restrict__ out, uint4* const* __restrict__ wtab) {
  const int64_t total = n * vec_per_row;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = t / vec_per_row;
    const int j = int(t - i * vec_per_row);
    const int peer = mode == 2 ? (self + 1 + int(i % (C - 1))) % C : (self + 1) % C;
    if (mode == 1) wtab[peer][int64_t(ids[i]) * vec_per_row + j] = out[t];               // push
    else out[t] = ld_nc_v4(tab[peer] + int64_t(ids[i]) * vec_per_row + j);               // pull / all-to-all
  }
}
__global__ void trial_collective_kernel(const float* const* __restrict__ tab, int C, int self, int mode, int64_t n,
                                        float* __restrict__ out) {
  // mode 0 all-gather (n floats per rank), 1 reduce-scatter (own chunk of n/C), 2 all-reduce (n)
  const int64_t chunk = mode == 1 ? n / C : n;
  const int64_t total = mode == 0 ? n * C : chunk;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    if (mode == 0) {
      out[t] = tab[t / n][t % n];
    } else {
      const int64_t j = mode == 1 ? int64_t(self) * chunk + t : t;
      float s = 0.f;
      for (int r = 0; r < C; ++r) s += tab[r][j];
      out[t] = s;
    }
  }
}
}  // namespace apt

extern "C" apt_status apt_profile_links(apt_ctx* c, apt_bw_profile* out) {
  if (!c || !out) return set_err(c, APT_E_INVALID, "apt_profile_links: bad arguments");
  memset(out, 0, sizeof *out);
  out->world = c->world;
  Arena A;
  const int64_t table_rows = 4 << 20, vec = 13;            // 4M rows x 208 B (products-like rows) = 872 MB
  uint4* table = A.alloc<uint4>(table_rows * vec, false);
  const int64_t n_big = 1 << 20, n_small = 1 << 12;
  int32_t* ids = A.alloc<int32_t>(n_big, false);
  uint4* outb = A.alloc<uint4>(n_big * vec, false);
  if (!table || !ids || !outb) return set_err(c, APT_E_OOM, "apt_profile_links: out of device memory");
  trial_ids_kernel<<<1024, 256, 0, c->stream>>>(ids, n_big, table_rows, 0x1234u);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto best = [&](auto&& launch) {
    float b = 1e30f;
    for (int it = 0; it < 6; ++it) {
      cudaEventRecord(e0, c->stream);
      launch();
      cudaEventRecord(e1, c->stream);
      cudaEventSynchronize(e1);
      float ms = 0.f;
      cudaEventElapsedTime(&ms, e0, e1);
      if (it) b = std::min(b, ms);   // first call warms up
    }
    return double(b) * 1e-3;
  };
  auto fit = [&](int op, double t_small, double b_small, double t_big, double b_big) {
    double beta = (b_big - b_small) / std::max(1e-12, t_big - t_small);
    double alpha = std::max(0.0, t_small - b_small / beta);
    out->alpha_s[op] = alpha;
    out->beta_Bps[op] = beta;
    out->measured[op] = 1;
  };
  const int blocks = num_sms() * 8;
  // local HBM gather: random rows of the table (the store's local tier)
  const double tg_s = best([&] { trial_gather_kernel<<<blocks, 256, 0, c->stream>>>(table, table_rows, vec, ids, n_small, outb); });
  const double tg_b = best([&] { trial_gather_kernel<<<blocks, 256, 0, c->stream>>>(table, table_rows, vec, ids, n_big, outb); });
  fit(APT_OP_LOCAL_GATHER, tg_s, double(n_small) * vec * 16, tg_b, double(n_big) * vec * 16);
  // host gather (pinned host memory read over PCIe/C2C): a device copy from pinned memory
  {
    void* hbuf = nullptr;
    if (cudaMallocHost(&hbuf, size_t(64) << 20) == cudaSuccess) {
      const double th_s = best([&] { cudaMemcpyAsync(outb, hbuf, size_t(1) << 16, cudaMemcpyHostToDevice, c->stream); });
      const double th_b = best([&] { cudaMemcpyAsync(outb, hbuf, size_t(64) << 20, cudaMemcpyHostToDevice, c->stream); });
      fit(APT_OP_HOST_GATHER, th_s, double(1 << 16), th_b, double(64 << 20));
      cudaFreeHost(hbuf);
    }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  CK(c, cudaGetLastError());
  // NVLink operators (peer pull / push, all-to-all, all-gather, reduce-scatter,
  // all-reduce): measured references of this pool (B200_PROFILING.md) when no peer
  // GPU is attached to this ctx ...
  const double nvl = 770e9, ar_bus = 725e9, a_peer = 3e-6;
  const int C = std::max(2, c->world);
  for (int op : {APT_OP_PEER_PULL, APT_OP_PEER_PUSH, APT_OP_ALLTOALLV, APT_OP_ALLGATHER, APT_OP_REDUCE_SCATTER,
                 APT_OP_ALLREDUCE}) {
    out->alpha_s[op] = a_peer;
    out->beta_Bps[op] = op == APT_OP_ALLREDUCE ? ar_bus * C / (2.0 * (C - 1)) : nvl;
    out->measured[op] = 0;
  }
  // ... and timed over the peers' CUDA-IPC-mapped tables in a job of one process per
  // GPU (collective: every rank runs the same trials between device barriers, so the
  // links carry all ranks' traffic at once, as in a step)
  if (multiprocess(c)) {
    std::vector<void*> opened;
    std::vector<void*> tv(c->world, nullptr);
    apt_status st = share_ptr(c, table, tv.data(), &opened);
    if (st != APT_OK) return st;
    uint4** tab = A.alloc<uint4*>(c->world, false);
    if (!tab) return set_err(c, APT_E_OOM, "apt_profile_links: out of device memory");
    CK(c, cudaMemcpyAsync(tab, tv.data(), sizeof(void*) * c->world, cudaMemcpyHostToDevice, c->stream));
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int self = c->rank, W = c->world;
    auto timed = [&](auto&& launch) -> double {   // barrier, then the op on every rank at once
      float b = 1e30f;
      for (int it = 0; it < 6; ++it) {
        if (device_barrier(c) != APT_OK) return -1.0;
        cudaEventRecord(e0, c->stream);
        launch();
        cudaEventRecord(e1, c->stream);
        cudaEventSynchronize(e1);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        if (it) b = std::min(b, ms);
      }
      return double(b) * 1e-3;
    };
    uint4* const* wtab = tab;
    const int modes[3] = {0, 1, 2};
    const int ops[3] = {APT_OP_PEER_PULL, APT_OP_PEER_PUSH, APT_OP_ALLTOALLV};
    for (int m = 0; m < 3; ++m) {
      const double ts = timed([&] { trial_peer_gather_kernel<<<blocks, 256, 0, c->stream>>>(tab, W, self, modes[m], table_rows, vec, ids, n_small, outb, wtab); });
      const double tb = timed([&] { trial_peer_gather_kernel<<<blocks, 256, 0, c->stream>>>(tab, W, self, modes[m], table_rows, vec, ids, n_big, outb, wtab); });
      if (ts < 0 || tb < 0) return set_err(c, APT_E_DEVICE_ASSERT, "apt_profile_links: barrier failed");
      fit(ops[m], ts, double(n_small) * vec * 16, tb, double(n_big) * vec * 16);
    }
    const float* const* ftab = reinterpret_cast<float* const*>(tab);
    float* fout = reinterpret_cast<float*>(outb);
    const int cops[3] = {APT_OP_ALLGATHER, APT_OP_REDUCE_SCATTER, APT_OP_ALLREDUCE};
    const int64_t f_small = int64_t(1) << 14, f_big = int64_t(1) << 22;   // floats per rank
    for (int m = 0; m < 3; ++m) {
      const double ts = timed([&] { trial_collective_kernel<<<blocks, 256, 0, c->stream>>>(ftab, W, self, m, f_small, fout); });
      const double tb = timed([&] { trial_collective_kernel<<<blocks, 256, 0, c->stream>>>(ftab, W, self, m, f_big, fout); });
      if (ts < 0 || tb < 0) return set_err(c, APT_E_DEVICE_ASSERT, "apt_profile_links: barrier failed");
      // bytes each rank receives: all-gather (C-1) n, reduce-scatter (C-1) n / C, all-reduce (C-1) n
      const double k = m == 1 ? double(W - 1) / W : double(W - 1);
      fit(cops[m], ts, 4.0 * f_small * k, tb, 4.0 * f_big * k);
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    CK(c, cudaStreamSynchronize(c->stream));
    if ((st = device_barrier(c)) != APT_OK) return st;
    CK(c, cudaStreamSynchronize(c->stream));
    close_peers(opened);
    char x = 0;
    std::vector<char> xs(c->world);
    if ((st = allgather(c, &x, xs.data(), 1)) != APT_OK) return st;   // every mapping closed before any free
  }
  return APT_OK;
}
