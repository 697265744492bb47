// runtime.cu -- C ABI (include/apt.h): contexts, graph, feature store,
// sampling batches and the single-op entry points.  The trainer (strategy
// drivers) is in trainer.cu, the planner in plan.cu.
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cmath>
#include <numeric>

#include "common.cuh"
#include "runtime.h"

using namespace apt;

namespace apt {
thread_local std::string g_err;

apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  if (c) c->err = buf;
  g_err = buf;
  return s;
}

void release_exported(apt_ctx* c);

static void ctx_free(apt_ctx* c) {
  cudaStreamSynchronize(c->stream);
  release_exported(c);
  if (c->side) { cudaStreamSynchronize(c->side); cudaStreamDestroy(c->side); }
  if (c->samp) { cudaStreamSynchronize(c->samp); cudaStreamDestroy(c->samp); }
  if (c->samp2) { cudaStreamSynchronize(c->samp2); cudaStreamDestroy(c->samp2); }
  if (c->ev_sfork) cudaEventDestroy(c->ev_sfork);
  if (c->ev_sjoin) cudaEventDestroy(c->ev_sjoin);
  if (c->tap) { cudaStreamSynchronize(c->tap); cudaStreamDestroy(c->tap); }
  if (c->ev_tap) cudaEventDestroy(c->ev_tap);
  if (c->ev_tapj) cudaEventDestroy(c->ev_tapj);
  if (c->ev_pfork) cudaEventDestroy(c->ev_pfork);
  if (c->ev_pjoin) cudaEventDestroy(c->ev_pjoin);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->ev_csc) cudaEventDestroy(c->ev_csc);
  c->arena.release();
  if (c->own_stream) cudaStreamDestroy(c->stream);
  delete c;
}
void ctx_retain(apt_ctx* c) { if (c) ++c->children; }
void ctx_release(apt_ctx* c) {
  if (c && --c->children == 0 && c->zombie) ctx_free(c);
}

apt_status check_cuda(apt_ctx* c, cudaError_t e, const char* what) {
  if (e == cudaSuccess) return APT_OK;
  if (c) c->broken = true;
  return set_err(c, APT_E_CUDA, "%s: %s", what, cudaGetErrorString(e));
}
}  // namespace apt

#define CK(ctx, expr)                                               \
  do {                                                              \
    apt_status _s = ::apt::check_cuda((ctx), (expr), #expr);        \
    if (_s != APT_OK) return _s;                                    \
  } while (0)

namespace apt {
apt_status fstore_create_p163(apt_ctx* c, const apt_graph* g, apt_strategy layout, apt_dtype dtype, int dim,
                              const float* host_feats, uint64_t feat_seed, const apt_fstore_opts* opts, apt_fstore** out);
}

extern "C" {

apt_status apt_ctx_create(int rank, int world, int device, void* stream, apt_ctx** out) {
  if (!out || world < 1 || world > APT_MAX_RANKS || rank < -1 || rank >= world)
    return set_err(nullptr, APT_E_INVALID, "apt_ctx_create: bad rank/world (%d/%d)", rank, world);
  auto* c = new apt_ctx();
  c->world = world;
  c->emulated = rank < 0;
  c->rank = rank < 0 ? 0 : rank;
  c->n_local = rank < 0 ? world : 1;
  c->device = device;
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) {
    set_err(nullptr, APT_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(e));
    delete c;
    return APT_E_CUDA;
  }
  int major = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device);
  cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, device);
  if (major != 10) {
    set_err(nullptr, APT_E_UNSUPPORTED, "device %d is sm_%d0: this library is built for sm_100a only", device, major);
    delete c;
    return APT_E_UNSUPPORTED;
  }
  // priorities: the step's chain and its side branch high, the next step's sampling
  // (pipelined trainer) at the lowest priority so it only fills idle SM slots
  int prio_lo = 0, prio_hi = 0;
  cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  if (stream) {
    c->stream = static_cast<cudaStream_t>(stream);
  } else {
    cudaStreamCreateWithPriority(&c->stream, cudaStreamNonBlocking, prio_hi);
    c->own_stream = true;
  }
  cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, prio_hi);
  // APT_SAMP_PRIO=1: the sampling stream at the chain's priority (A/B)
  static const int samp_hi = [] { const char* v = std::getenv("APT_SAMP_PRIO"); return v ? atoi(v) : 0; }();
  cudaStreamCreateWithPriority(&c->samp, cudaStreamNonBlocking, samp_hi ? prio_hi : prio_lo);
  cudaStreamCreateWithPriority(&c->tap, cudaStreamNonBlocking, prio_hi);
  // APT_SAMP2_PRIO=1: the background block transposes at the chain's priority (A/B)
  static const int samp2_hi = [] { const char* v = std::getenv("APT_SAMP2_PRIO"); return v ? atoi(v) : 0; }();
  cudaStreamCreateWithPriority(&c->samp2, cudaStreamNonBlocking, (samp_hi || samp2_hi) ? prio_hi : prio_lo);
  cudaEventCreateWithFlags(&c->ev_sfork, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_sjoin, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_tap, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_tapj, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_pfork, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_pjoin, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&c->ev_csc, cudaEventDisableTiming);
  c->dev_err = c->arena.alloc<uint32_t>(4);
  c->scratch = c->arena.alloc<int32_t>(16);
  if (!c->dev_err || !c->scratch) {
    delete c;
    return set_err(nullptr, APT_E_OOM, "apt_ctx_create: out of device memory");
  }
  *out = c;
  return APT_OK;
}

apt_status apt_ctx_destroy(apt_ctx* c) {
  if (!c) return APT_OK;
  if (c->children > 0) {
    c->zombie = true;   // released with its last child
    return APT_OK;
  }
  apt::ctx_free(c);
  return APT_OK;
}

const char* apt_last_error(const apt_ctx* c) { return c ? c->err.c_str() : g_err.c_str(); }

int64_t apt_ctx_launches(const apt_ctx* c) { return c ? c->launches : 0; }

apt_status apt_ctx_sync(apt_ctx* c) {
  if (!c) return set_err(nullptr, APT_E_INVALID, "null ctx");
  CK(c, cudaStreamSynchronize(c->stream));
  uint32_t w = 0;
  CK(c, cudaMemcpy(&w, c->dev_err, 4, cudaMemcpyDeviceToHost));
  if (w) return set_err(c, APT_E_DEVICE_ASSERT, "device error word 0x%x", w);
  return APT_OK;
}

apt_status apt_memcpy(apt_ctx* c, void* dst, const void* src, size_t bytes, int kind) {
  if (!c || (!dst && bytes) || (!src && bytes)) return set_err(c, APT_E_INVALID, "apt_memcpy: null");
  cudaMemcpyKind k = kind == 0 ? cudaMemcpyDeviceToHost : kind == 1 ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  CK(c, cudaMemcpyAsync(dst, src, bytes, k, c->stream));
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

// ------------------------------------------------------------------ graph
apt_status apt_graph_load(apt_ctx* c, int64_t n, int64_t nnz, const int64_t* indptr, const int32_t* indices,
                          const int32_t* part, apt_graph** out) {
  if (!c || !out || n <= 0 || nnz < 0 || !indptr || (!indices && nnz))
    return set_err(c, APT_E_INVALID, "apt_graph_load: bad arguments");
  if (n >= (int64_t(1) << 31)) return set_err(c, APT_E_INVALID, "apt_graph_load: n_nodes >= 2^31");
  if (indptr[0] != 0 || indptr[n] != nnz) return set_err(c, APT_E_INVALID, "apt_graph_load: indptr[0]/indptr[n] mismatch");
  auto* g = new apt_graph();
  g->ctx = c;
  ctx_retain(c);
  g->n = n;
  g->nnz = nnz;
  g->world = c->world;
  g->indptr = g->arena.alloc<int64_t>(n + 1, false);
  g->indices = g->arena.alloc<int32_t>(nnz, false);
  g->part = g->arena.alloc<int32_t>(n, false);
  g->lrow = g->arena.alloc<int32_t>(n, false);
  g->loc = g->arena.alloc<int2>(n, false);
  if (!g->indptr || !g->indices || !g->part || !g->lrow || !g->loc) {
    apt_graph_destroy(g);
    return set_err(c, APT_E_OOM, "apt_graph_load: out of device memory (n=%lld nnz=%lld)", (long long)n, (long long)nnz);
  }
  g->part_h.resize(n);
  std::vector<int32_t> lrow(n);
  g->shard_rows.assign(c->world, 0);
  for (int64_t u = 0; u < n; ++u) {
    int p = part ? part[u] : int((u * c->world) / n);
    if (p < 0 || p >= c->world) {
      apt_graph_destroy(g);
      return set_err(c, APT_E_INVALID, "apt_graph_load: part[%lld]=%d out of range", (long long)u, p);
    }
    g->part_h[u] = p;
    lrow[u] = int32_t(g->shard_rows[p]++);
  }
  CK(c, cudaMemcpyAsync(g->indptr, indptr, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, c->stream));
  if (nnz) CK(c, cudaMemcpyAsync(g->indices, indices, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, c->stream));
  CK(c, cudaMemcpyAsync(g->part, g->part_h.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice, c->stream));
  CK(c, cudaMemcpyAsync(g->lrow, lrow.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice, c->stream));
  {
    std::vector<int2> loc(n);
    for (int64_t u = 0; u < n; ++u) loc[u] = make_int2(g->part_h[u], lrow[u]);
    CK(c, cudaMemcpyAsync(g->loc, loc.data(), sizeof(int2) * n, cudaMemcpyHostToDevice, c->stream));
    CK(c, cudaStreamSynchronize(c->stream));
  }
  CK(c, cudaStreamSynchronize(c->stream));
  *out = g;
  return APT_OK;
}

apt_status apt_graph_destroy(apt_graph* g) {
  if (!g) return APT_OK;
  apt_ctx* c = g->ctx;
  delete g;
  ctx_release(c);
  return APT_OK;
}

// ------------------------------------------------------------- feature store
apt_status apt_fstore_create(apt_ctx* c, const apt_graph* g, apt_strategy layout, apt_dtype dtype, int dim,
                             const float* host_feats, uint64_t feat_seed, apt_fstore** out) {
  return apt_fstore_create_tiered(c, g, layout, dtype, dim, host_feats, feat_seed, nullptr, out);
}

apt_status apt_fstore_create_tiered(apt_ctx* c, const apt_graph* g, apt_strategy layout, apt_dtype dtype, int dim,
                                    const float* host_feats, uint64_t feat_seed, const apt_fstore_opts* opts,
                                    apt_fstore** out) {
  if (!c || !g || !out || dim <= 0 || (dtype != APT_F32 && dtype != APT_BF16) || layout < APT_GDP || layout > APT_AUTO)
    return set_err(c, APT_E_INVALID, "apt_fstore_create: bad arguments");
  if (opts && opts->cache_rule == APT_CACHE_P163) return apt::fstore_create_p163(c, g, layout, dtype, dim, host_feats,
                                                                                  feat_seed, opts, out);
  const double frac = opts ? opts->hbm_frac : 1.0;
  const int64_t want_cache = opts ? opts->cache_rows : 0;
  if (!(frac > 0.0 && frac <= 1.0) || want_cache < 0 || (want_cache > 0 && !opts->hot_ids))
    return set_err(c, APT_E_INVALID, "apt_fstore_create: hbm_frac in (0,1], cache_rows >= 0 with hot_ids");
  auto* f = new apt_fstore();
  f->ctx = c;
  ctx_retain(c);
  f->g = g;
  f->layout = layout == APT_AUTO ? APT_GDP : layout;
  f->dtype = dtype == APT_BF16 ? kBF16 : kF32;
  f->dim = dim;
  f->world = c->world;
  const int C = c->world;
  const bool col_sharded = f->layout == APT_NFP && C > 1;
  f->tiered = !col_sharded && (frac < 1.0 || want_cache > 0);
  f->hbm_frac = frac;
  if (col_sharded && (frac < 1.0 || want_cache > 0)) {
    apt_fstore_destroy(f);
    return set_err(c, APT_E_UNSUPPORTED, "apt_fstore_create: tiers apply to row-sharded stores (NFP reads only its "
                                         "column slice and has no excess cache, P:175-178)");
  }
  const int align = dtype == APT_BF16 ? 8 : 4;     // 16-byte rows
  const size_t esz = dtype == APT_BF16 ? 2 : 4;
  // ids of every shard's rows, ascending (a single shard holds every node)
  std::vector<std::vector<int32_t>> ids(C);
  if (!col_sharded) {
    if (C > 1) {
      for (int64_t u = 0; u < g->n; ++u) ids[g->part_h[u]].push_back(int32_t(u));
    } else {
      ids[0].resize(g->n);
      for (int64_t u = 0; u < g->n; ++u) ids[0][u] = int32_t(u);
    }
  }
  for (int r = 0; r < C; ++r) {
    if (col_sharded) {
      f->col_lo[r] = int((int64_t(r) * dim) / C);
      f->col_hi[r] = int((int64_t(r + 1) * dim) / C);
      f->rows[r] = g->n;
    } else {
      f->col_lo[r] = 0;
      f->col_hi[r] = dim;
      const int64_t all = int64_t(ids[r].size());
      f->rows[r] = std::min<int64_t>(all, int64_t(std::ceil(frac * double(all))));   // rows kept in HBM
    }
    const int w = std::max(1, f->col_hi[r] - f->col_lo[r]);
    f->pitch[r] = round_up(w, align);
  }
  const int64_t pitch = f->pitch[0];
  int32_t* ids_dev = f->arena.alloc<int32_t>(std::max<int64_t>(g->n, 1), false);
  auto fill_rows = [&](void* dst, const int32_t* ids_h, int64_t n_rows, int col0, int ncols, int64_t pch) -> apt_status {
    if (n_rows <= 0) return APT_OK;
    if (host_feats) {
      std::vector<uint8_t> buf(size_t(n_rows * pch) * esz, 0);
      for (int64_t i = 0; i < n_rows; ++i) {
        const int64_t u = ids_h ? ids_h[i] : i;
        for (int j = 0; j < ncols; ++j) {
          const float v = host_feats[u * dim + col0 + j];
          if (esz == 4) {
            reinterpret_cast<float*>(buf.data())[i * pch + j] = v;
          } else {
            uint32_t bits;
            memcpy(&bits, &v, 4);
            bits = (bits + 0x7FFFu + ((bits >> 16) & 1u)) >> 16;   // RNE
            reinterpret_cast<uint16_t*>(buf.data())[i * pch + j] = uint16_t(bits);
          }
        }
      }
      CK(c, cudaMemcpyAsync(dst, buf.data(), buf.size(), cudaMemcpyDefault, c->stream));
    } else {
      const int32_t* idp = nullptr;
      if (ids_h) {
        CK(c, cudaMemcpyAsync(ids_dev, ids_h, sizeof(int32_t) * n_rows, cudaMemcpyHostToDevice, c->stream));
        idp = ids_dev;
      }
      CK(c, launch_fill_features(dst, f->dtype, pch, col0, ncols, idp, n_rows, feat_seed, c->stream));
      c->launches++;
    }
    CK(c, cudaStreamSynchronize(c->stream));
    return APT_OK;
  };
  for (int r = 0; r < C; ++r) {
    // emulated: all shards here; multi-process: only the own shard is local
    if (!c->emulated && r != c->rank) continue;
    // one zero-filled row past the shard's rows: padding edges of the layer-1 gather read
    // it (FeatView::zrow), so every load of a batch is a plain global load
    f->shard[r] = f->arena.alloc<uint8_t>((f->rows[r] + 1) * f->pitch[r] * int64_t(esz), true);
    if (!f->shard[r] || !ids_dev) {
      apt_fstore_destroy(f);
      return set_err(c, APT_E_OOM, "apt_fstore_create: out of device memory");
    }
    const int ncols = f->col_hi[r] - f->col_lo[r];
    apt_status st = col_sharded ? fill_rows(f->shard[r], nullptr, f->rows[r], f->col_lo[r], ncols, f->pitch[r])
                                : fill_rows(f->shard[r], C > 1 ? ids[r].data() : nullptr, f->rows[r], 0, ncols,
                                            f->pitch[r]);
    if (st != APT_OK) { apt_fstore_destroy(f); return st; }
  }
  if (f->tiered) {
    // host tier: every shard's rows beyond its HBM budget, in (owner, row) order; each
    // process keeps the whole tier in its pinned host memory (like the topology)
    std::vector<int32_t> host_ids;
    for (int r = 0; r < C; ++r)
      for (size_t i = size_t(f->rows[r]); i < ids[r].size(); ++i) host_ids.push_back(ids[r][i]);
    f->host_rows = int64_t(host_ids.size());
    if (f->host_rows > 0) {
      if (cudaHostAlloc(&f->host, size_t(f->host_rows * pitch) * esz, cudaHostAllocMapped | cudaHostAllocPortable) !=
          cudaSuccess) {
        apt_fstore_destroy(f);
        return set_err(c, APT_E_OOM, "apt_fstore_create: pinned host tier of %lld rows", (long long)f->host_rows);
      }
      apt_status st = fill_rows(f->host, host_ids.data(), f->host_rows, 0, dim, pitch);
      if (st != APT_OK) { apt_fstore_destroy(f); return st; }
    }
    std::vector<int32_t> base_tier(g->n), base_row(g->n);
    for (int r = 0; r < C; ++r)
      for (size_t i = 0; i < ids[r].size(); ++i) {
        const int32_t u = ids[r][i];
        if (int64_t(i) < f->rows[r]) { base_tier[u] = r; base_row[u] = int32_t(i); }
        else { base_tier[u] = C; base_row[u] = -1; }
      }
    for (int64_t i = 0, h = 0; i < int64_t(host_ids.size()); ++i, ++h) base_row[host_ids[i]] = int32_t(h);
    // HBM rows per shard + every rank's cache membership (dry-run classification)
    f->rows_dev = f->arena.alloc<int64_t>(C, false);
    CK(c, cudaMemcpyAsync(f->rows_dev, f->rows, sizeof(int64_t) * C, cudaMemcpyHostToDevice, c->stream));
    const int64_t n_words = ceil_div(g->n, 32);
    if (want_cache > 0) {
      std::vector<uint32_t> bm(size_t(C) * n_words, 0u);
      for (int r = 0; r < C; ++r) {
        int64_t taken = 0;
        for (int64_t j = 0; j < want_cache && taken < want_cache; ++j) {
          const int64_t u = opts->hot_ids[j];
          if (u < 0 || u >= g->n) { apt_fstore_destroy(f); return set_err(c, APT_E_INVALID, "hot id out of range"); }
          uint32_t& w = bm[size_t(r) * n_words + (u >> 5)];
          if (base_tier[u] == r || (w >> (u & 31) & 1u)) continue;
          w |= 1u << (u & 31);
          ++taken;
        }
      }
      f->cache_bm = f->arena.alloc<uint32_t>(int64_t(C) * n_words, false);
      if (!f->cache_bm) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "cache bitmaps"); }
      CK(c, cudaMemcpyAsync(f->cache_bm, bm.data(), sizeof(uint32_t) * bm.size(), cudaMemcpyHostToDevice, c->stream));
    }
    CK(c, cudaStreamSynchronize(c->stream));
    // per hosted rank: its view, with its cache of hot rows (those it does not hold in HBM)
    for (int r = 0; r < C; ++r) {
      if (!c->emulated && r != c->rank) continue;
      std::vector<int32_t> tier = base_tier, trow = base_row, cached;
      for (int64_t j = 0; j < want_cache && int64_t(cached.size()) < want_cache; ++j) {
        const int64_t u = opts->hot_ids[j];
        if (u < 0 || u >= g->n) { apt_fstore_destroy(f); return set_err(c, APT_E_INVALID, "hot id out of range"); }
        if (tier[u] == r || tier[u] == C + 1) continue;          // already local
        tier[u] = C + 1;
        trow[u] = int32_t(cached.size());
        cached.push_back(int32_t(u));
      }
      f->cache_rows[r] = int64_t(cached.size());
      if (!cached.empty()) {
        f->cache[r] = f->arena.alloc<uint8_t>(f->cache_rows[r] * pitch * int64_t(esz), false);
        if (!f->cache[r]) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "apt_fstore_create: cache"); }
        apt_status st = fill_rows(f->cache[r], cached.data(), f->cache_rows[r], 0, dim, pitch);
        if (st != APT_OK) { apt_fstore_destroy(f); return st; }
      }
      f->loc_map[r] = f->arena.alloc<int2>(g->n, false);
      if (!f->loc_map[r]) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "feature map"); }
      {
        std::vector<int2> loc(g->n);
        for (int64_t u = 0; u < g->n; ++u) loc[u] = make_int2(tier[u], trow[u]);
        CK(c, cudaMemcpyAsync(f->loc_map[r], loc.data(), sizeof(int2) * g->n, cudaMemcpyHostToDevice, c->stream));
        CK(c, cudaStreamSynchronize(c->stream));
      }
      f->tier_h[r] = std::move(tier);
    }
  }
  if (multiprocess(c) && !col_sharded) {
    // row-sharded store: every rank maps every peer's shard (GDP / DNP halo reads over NVLink)
    void* tab[APT_MAX_RANKS] = {};
    apt_status s = share_ptr(c, f->shard[c->rank], tab, &f->peer_opened);
    if (s != APT_OK) { apt_fstore_destroy(f); return s; }
    for (int r = 0; r < C; ++r) f->shard[r] = tab[r];
  }
  *out = f;
  return APT_OK;
}

apt_status apt_fstore_destroy(apt_fstore* f) {
  if (!f) return APT_OK;
  apt_ctx* c = f->ctx;
  delete f;
  ctx_release(c);
  return APT_OK;
}

}  // extern "C"

namespace apt {
// FeatView of the row-sharded store as seen by rank r (every shard reachable:
// locally or through its peer pointer).
FeatView feat_view(const apt_fstore* f, int r) {
  FeatView v{};
  v.zrow = -1;
  const bool rows_sharded = f->layout != APT_NFP && f->world > 1;
  for (int o = 0; o < f->world; ++o) v.base[o] = f->shard[o];
  if (f->tiered) {
    const int rr = f->world > 1 ? r : 0;
    v.base[f->world] = f->host;
    v.base[f->world + 1] = f->cache[rr];
    v.loc = f->loc_map[rr];
    v.pitch = f->pitch[0];
    v.dim = f->dim;
  } else if (rows_sharded) {
    v.loc = f->g->loc;
    v.pitch = f->pitch[0];
    v.dim = f->dim;
  } else {
    const int s = f->world > 1 ? r : 0;
    v.base[0] = f->shard[s];
    v.loc = nullptr;
    v.pitch = f->pitch[s];
    v.dim = f->col_hi[s] - f->col_lo[s];
    v.zrow = f->rows[s];
  }
  v.col0 = 0;
  v.dtype = f->dtype;
  return v;
}
}  // namespace apt

extern "C" {

// ---------------------------------------------------------------- sampling
apt_status apt_sample(apt_ctx* c, const apt_graph* g, const int64_t* seeds_dev, int64_t n_seeds,
                      const int32_t* fanouts, int K, uint64_t rng_seed, uint64_t step, apt_batch** out) {
  if (!c || !g || !out || (!seeds_dev && n_seeds) || n_seeds < 0 || !fanouts || K < 1 || K > APT_MAX_LAYERS)
    return set_err(c, APT_E_INVALID, "apt_sample: bad arguments");
  for (int l = 0; l < K; ++l)
    if (fanouts[l] < 1 || fanouts[l] > 256) return set_err(c, APT_E_INVALID, "apt_sample: fanout %d out of [1,256]", fanouts[l]);
  auto* b = new apt_batch();
  b->ctx = c;
  ctx_retain(c);
  b->K = K;
  b->g = g;
  b->rng_seed = rng_seed;
  b->step = step;
  for (int l = 0; l < K; ++l) b->fanouts[l] = fanouts[l];
  const int64_t n_words = ceil_div(g->n, 32);
  uint32_t* dst_bm = b->arena.alloc<uint32_t>(n_words, true);
  uint32_t* new_bm = b->arena.alloc<uint32_t>(n_words, true);
  int32_t* pos = b->arena.alloc<int32_t>(g->n, false);
  int64_t maxF = n_seeds;
  int64_t max_part = 2 * ceil_div(n_words, kScanWsTile) + 8;
  int32_t* counts = b->arena.alloc<int32_t>(4 * K + 4, true);
  uint64_t* step_dev = b->arena.alloc<uint64_t>(1, false);
  int32_t* seeds32 = b->arena.alloc<int32_t>(n_seeds, false);
  if (!dst_bm || !new_bm || !pos || !counts || !step_dev || !seeds32) {
    apt_batch_destroy(b);
    return set_err(c, APT_E_OOM, "apt_sample: out of device memory");
  }
  // int64 seeds -> int32 (validated on the host copy)
  {
    std::vector<int64_t> h(n_seeds);
    CK(c, cudaMemcpyAsync(h.data(), seeds_dev, sizeof(int64_t) * n_seeds, cudaMemcpyDeviceToHost, c->stream));
    CK(c, cudaStreamSynchronize(c->stream));
    std::vector<int32_t> h32(n_seeds);
    for (int64_t i = 0; i < n_seeds; ++i) {
      if (h[i] < 0 || h[i] >= g->n) {
        apt_batch_destroy(b);
        return set_err(c, APT_E_INVALID, "apt_sample: seed %lld out of range", (long long)h[i]);
      }
      h32[i] = int32_t(h[i]);
    }
    int32_t ns = int32_t(n_seeds);
    CK(c, cudaMemcpyAsync(seeds32, h32.data(), sizeof(int32_t) * n_seeds, cudaMemcpyHostToDevice, c->stream));
    CK(c, cudaMemcpyAsync(counts, &ns, 4, cudaMemcpyHostToDevice, c->stream));
    CK(c, cudaMemcpyAsync(step_dev, &step, 8, cudaMemcpyHostToDevice, c->stream));
  }
  const int32_t* dst = seeds32;
  const int32_t* n_dst = counts;   // counts[0] = n_seeds; counts[1+2h] = n_src(h), counts[2+2h] = n_edges(h)
  int32_t* partials = b->arena.alloc<int32_t>(max_part, false);
  for (int h = 0; h < K; ++h) {
    const int k = fanouts[K - 1 - h];
    const int64_t maxS = std::max<int64_t>(maxF, std::min<int64_t>(maxF * (1 + k), g->n));
    int32_t* cnt = b->arena.alloc<int32_t>(maxF, true);
    int32_t* nbr = b->arena.alloc<int32_t>(maxF * k, false);
    int32_t* src = b->arena.alloc<int32_t>(maxS, false);
    int32_t* indptr = b->arena.alloc<int32_t>(maxF + 1, true);
    int32_t* indices = b->arena.alloc<int32_t>(maxF * k, false);
    int32_t* part2 = b->arena.alloc<int32_t>(2 * ceil_div(maxF, kScanWsTile) + 8, false);
    if (!cnt || !nbr || !src || !indptr || !indices || !partials || !part2) {
      apt_batch_destroy(b);
      return set_err(c, APT_E_OOM, "apt_sample: out of device memory");
    }
    SampleArgs sa{g->indptr, g->indices, dst, n_dst, maxF, k, philox_key(rng_seed, kDomSample), step_dev, h, cnt, nbr};
    CK(c, launch_sample(sa, c->stream));
    CompactArgs ca{dst, n_dst, maxF, cnt, nbr, k, dst_bm, new_bm, n_words, pos, src, counts + 1 + 2 * h,
                   indptr, indices, counts + 2 + 2 * h, partials, part2};
    CK(c, launch_compact(ca, c->stream));
    c->launches += 4;
    b->dst[h] = const_cast<int32_t*>(dst);
    b->src[h] = src;
    b->indptr[h] = indptr;
    b->indices[h] = indices;
    b->cnt[h] = cnt;
    b->nbr[h] = nbr;
    dst = src;
    n_dst = counts + 1 + 2 * h;
    maxF = maxS;
  }
  std::vector<int32_t> hc(4 * K + 4);
  CK(c, cudaMemcpyAsync(hc.data(), counts, sizeof(int32_t) * hc.size(), cudaMemcpyDeviceToHost, c->stream));
  CK(c, cudaStreamSynchronize(c->stream));
  int64_t nd = n_seeds;
  b->counts = counts;
  for (int h = 0; h < K; ++h) {
    b->n_dst[h] = nd;
    b->n_src[h] = hc[1 + 2 * h];
    b->n_edges[h] = hc[2 + 2 * h];
    nd = b->n_src[h];
    // int64 ids at the ABI (apt_block_view): widened once here
    b->dst64[h] = b->arena.alloc<int64_t>(b->n_dst[h], false);
    b->src64[h] = b->arena.alloc<int64_t>(b->n_src[h], false);
    if (!b->dst64[h] || !b->src64[h]) {
      apt_batch_destroy(b);
      return set_err(c, APT_E_OOM, "apt_sample: out of device memory");
    }
    CK(c, launch_widen_ids(b->dst[h], b->n_dst[h], b->dst64[h], c->stream));
    CK(c, launch_widen_ids(b->src[h], b->n_src[h], b->src64[h], c->stream));
    c->launches += 2;
  }
  CK(c, cudaStreamSynchronize(c->stream));
  *out = b;
  return APT_OK;
}

apt_status apt_batch_group(apt_ctx* c, const apt_batch* const* per_rank, int n, apt_batch** out) {
  if (!c || !per_rank || !out || n < 1 || n > APT_MAX_RANKS || n != c->n_local)
    return set_err(c, APT_E_INVALID, "apt_batch_group: need one batch per hosted rank (%d)", c ? c->n_local : 0);
  for (int i = 0; i < n; ++i) {
    const apt_batch* m = per_rank[i];
    if (!m || m->ctx != c || !m->members.empty() || m->K != per_rank[0]->K || m->g != per_rank[0]->g ||
        m->rng_seed != per_rank[0]->rng_seed || m->step != per_rank[0]->step)
      return set_err(c, APT_E_INVALID, "apt_batch_group: batch %d is not a plain batch of this ctx with the same "
                                       "graph, K, rng_seed and step", i);
    for (int l = 0; l < m->K; ++l)
      if (m->fanouts[l] != per_rank[0]->fanouts[l]) return set_err(c, APT_E_INVALID, "apt_batch_group: fanouts differ");
  }
  auto* b = new apt_batch();
  b->ctx = c;
  ctx_retain(c);
  b->g = per_rank[0]->g;
  b->K = per_rank[0]->K;
  b->rng_seed = per_rank[0]->rng_seed;
  b->step = per_rank[0]->step;
  for (int l = 0; l < b->K; ++l) b->fanouts[l] = per_rank[0]->fanouts[l];
  b->members.assign(per_rank, per_rank + n);
  *out = b;
  return APT_OK;
}

apt_status apt_batch_block(const apt_batch* b, int hop, apt_block_view* out) {
  if (!b || !out || hop < 0 || hop >= b->K) return set_err(nullptr, APT_E_INVALID, "apt_batch_block: bad hop");
  if (!b->members.empty()) return set_err(b->ctx, APT_E_INVALID, "apt_batch_block: a batch group has no single block");
  out->n_dst = b->n_dst[hop];
  out->n_src = b->n_src[hop];
  out->n_edges = b->n_edges[hop];
  out->dst_ids = b->dst64[hop];
  out->src_ids = b->src64[hop];
  out->indptr = b->indptr[hop];
  out->indices = b->indices[hop];
  return APT_OK;
}

apt_status apt_batch_destroy(apt_batch* b) {
  if (!b) return APT_OK;
  apt_ctx* c = b->ctx;
  delete b;
  ctx_release(c);
  return APT_OK;
}

// ------------------------------------------------------------- single ops
apt_status apt_gather(apt_ctx* c, const apt_fstore* f, const int64_t* ids, int64_t n, void* out) {
  if (!c || !f || (n && (!ids || !out)) || n < 0) return set_err(c, APT_E_INVALID, "apt_gather: bad arguments");
  if (!n) return APT_OK;
  FeatView v = feat_view(f, c->rank);
  // int64 ids at the ABI, int32 inside: narrowed on the device, an id
  // outside [0, n_nodes) sets the device error word (APT_E_DEVICE_ASSERT at the next sync)
  int32_t* ids32 = nullptr;
  CK(c, cudaMallocAsync(&ids32, sizeof(int32_t) * n, c->stream));
  CK(c, launch_narrow_ids(ids, n, f->g->n, ids32, c->dev_err, c->stream));
  CK(c, launch_gather(v, ids32, nullptr, n, out, v.pitch, c->stream));
  CK(c, cudaFreeAsync(ids32, c->stream));
  c->launches += 2;
  return APT_OK;
}

apt_status apt_aggregate(apt_ctx* c, const apt_block_view* blk, const void* x, apt_dtype dt, int dim, int64_t x_pitch,
                         float* z, int64_t z_pitch) {
  if (!c || !blk || !x || !z || dim <= 0 || x_pitch < dim || z_pitch < dim || (z_pitch % 4) || dt != APT_F32)
    return set_err(c, APT_E_INVALID, "apt_aggregate: bad arguments (fp32 x, pitches multiple of 4)");
  if (x_pitch % 4) return set_err(c, APT_E_INVALID, "apt_aggregate: x_pitch must be a multiple of 4");
  int32_t* nd = c->scratch;
  int32_t h = int32_t(blk->n_dst);
  CK(c, cudaMemcpyAsync(nd, &h, 4, cudaMemcpyHostToDevice, c->stream));
  AggArgs a{};
  a.indptr = blk->indptr;
  a.indices = blk->indices;
  a.x = static_cast<const float*>(x);
  a.x_pitch = x_pitch;
  a.n_dst = nd;
  a.max_dst = blk->n_dst;
  a.dim = dim;
  a.z_f32 = z;
  a.z_f32_pitch = z_pitch;
  CK(c, launch_agg_csr(a, c->stream));
  c->launches++;
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

apt_status apt_aggregate_bwd(apt_ctx* c, const apt_block_view* blk, const float* dz, int dim, int64_t dz_pitch,
                             float* dx, int64_t dx_pitch) {
  if (!c || !blk || !dz || !dx || dim <= 0 || (dz_pitch % 4) || (dx_pitch % 4))
    return set_err(c, APT_E_INVALID, "apt_aggregate_bwd: bad arguments");
  int32_t* nd = c->scratch;
  int32_t h = int32_t(blk->n_dst);
  CK(c, cudaMemcpyAsync(nd, &h, 4, cudaMemcpyHostToDevice, c->stream));
  CK(c, launch_agg_bwd(blk->indptr, blk->indices, nd, blk->n_dst, dz, dz_pitch, dim, dx, dx_pitch, c->stream));
  c->launches++;
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

apt_status apt_project(apt_ctx* c, const void* Z, int64_t z_pitch, apt_dtype dt, const float* W, const float* bias,
                       int64_t M, int N, int K, int relu, float* Y, int64_t y_pitch) {
  if (!c || !Z || !W || !Y || M < 0 || N <= 0 || K <= 0 || z_pitch < K || y_pitch < N)
    return set_err(c, APT_E_INVALID, "apt_project: bad arguments");
  int32_t* md = c->scratch;
  int32_t mh = int32_t(M);
  CK(c, cudaMemcpyAsync(md, &mh, 4, cudaMemcpyHostToDevice, c->stream));
  if (dt == APT_BF16) {
    const int64_t wp = round_up(K, 8);
    uint16_t* Wb = nullptr;
    CK(c, cudaMallocAsync(reinterpret_cast<void**>(&Wb), sizeof(uint16_t) * N * wp, c->stream));
    CK(c, cudaMemsetAsync(Wb, 0, sizeof(uint16_t) * N * wp, c->stream));
    CK(c, launch_to_bf16(W, K, Wb, wp, K, nullptr, N, c->stream));
    if (tc_gemm_supported(N, K)) {   // the row-tile kernel (resident W)
      TcGemmArgs a{static_cast<const uint16_t*>(Z), z_pitch, Wb, wp, M, md, N, K, bias, relu, Y, y_pitch,
                   nullptr, nullptr, nullptr, 0};
      CK(c, launch_tc_gemm(a, c->stream));
    } else {                         // wider: the general tcgen05 kernel (N tiled, K streamed)
      SimtGemmArgs a{};
      a.A = Z; a.a_t = kBF16; a.sam = z_pitch; a.sak = 1;
      a.B = Wb; a.b_t = kBF16; a.sbk = 1; a.sbn = wp;
      a.C = Y; a.ldc = y_pitch; a.bias = bias; a.M_dev = md; a.M = M; a.N = N; a.K = K; a.relu = relu;
      CK(c, launch_simt_gemm(a, c->stream));
    }
    CK(c, cudaFreeAsync(Wb, c->stream));
    c->launches += 2;
  } else {
    SimtGemmArgs a{};
    a.A = Z; a.a_t = kF32; a.sam = z_pitch; a.sak = 1;
    a.B = W; a.b_t = kF32; a.sbk = 1; a.sbn = K;
    a.C = Y; a.ldc = y_pitch; a.bias = bias; a.M_dev = md; a.M = M; a.N = N; a.K = K; a.relu = relu;
    CK(c, launch_simt_gemm(a, c->stream));
    c->launches++;
  }
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

apt_status apt_weight_grad(apt_ctx* c, const float* G, int64_t g_pitch, const void* Z, int64_t z_pitch, apt_dtype dt,
                           int64_t rows, int d_out, int d_in, float* dW, float* db) {
  if (!c || !G || !Z || !dW || rows < 0 || d_out <= 0 || d_in <= 0 || g_pitch < d_out || z_pitch < d_in ||
      (g_pitch % 4))
    return set_err(c, APT_E_INVALID, "apt_weight_grad: bad arguments");
  int32_t* rd = c->scratch;
  int32_t rh = int32_t(rows);
  CK(c, cudaMemcpyAsync(rd, &rh, 4, cudaMemcpyHostToDevice, c->stream));
  if (dt == APT_BF16) {
    // G -> bf16 (tail of the last 64-row block zeroed); Z -> a copy with the all-ones column d_in
    const int64_t gbp = round_up(d_out, 8), zbp = round_up(d_in + 1, 8);
    const int64_t rr = std::max<int64_t>(rows, 1);
    uint16_t *Gb = nullptr, *Zb = nullptr;
    CK(c, cudaMallocAsync(reinterpret_cast<void**>(&Gb), sizeof(uint16_t) * rr * gbp, c->stream));
    CK(c, cudaMallocAsync(reinterpret_cast<void**>(&Zb), sizeof(uint16_t) * rr * zbp, c->stream));
    CK(c, launch_grad_finish(G, g_pitch, nullptr, 0, d_out, 0, Gb, gbp, rd, rr, c->stream));
    CK(c, launch_bf16_pad_ones(static_cast<const uint16_t*>(Z), z_pitch, Zb, zbp, d_in, rd, rr, c->stream));
    float* dbw = db;
    if (!dbw) CK(c, cudaMallocAsync(reinterpret_cast<void**>(&dbw), sizeof(float) * d_out, c->stream));
    if (tc_wgrad_supported(d_out, d_in)) {
      TcWgradArgs w{Gb, gbp, Zb, zbp, rd, rr, d_out, d_in, dW, dbw};
      CK(c, launch_tc_wgrad(w, c->stream));
    } else {   // wider: the general tcgen05 kernel, db from Z's all-ones column
      SimtGemmArgs a{};
      a.A = Gb; a.a_t = kBF16; a.sam = 1; a.sak = gbp;
      a.B = Zb; a.b_t = kBF16; a.sbk = zbp; a.sbn = 1;
      a.C = dW; a.ldc = d_in; a.M = d_out; a.N = d_in + 1; a.K = rr; a.K_dev = rd; a.accumulate = 1;
      CK(c, launch_tc_gen_gemm(a, d_in, dbw, c->stream));
    }
    if (!db) CK(c, cudaFreeAsync(dbw, c->stream));
    CK(c, cudaFreeAsync(Gb, c->stream));
    CK(c, cudaFreeAsync(Zb, c->stream));
    c->launches += 3;
  } else {
    SimtGemmArgs a{};
    a.A = G; a.a_t = kF32; a.sam = 1; a.sak = g_pitch;
    a.B = Z; a.b_t = kF32; a.sbk = z_pitch; a.sbn = 1;
    a.C = dW; a.ldc = d_in; a.M = d_out; a.N = d_in; a.K = std::max<int64_t>(rows, 1); a.K_dev = rd;
    a.accumulate = 1; a.k_chunk = 2048;
    CK(c, launch_simt_gemm(a, c->stream));   // 3xTF32 tensor cores when TMA-addressable
    if (db) CK(c, launch_colsum(G, g_pitch, d_out, rd, std::max<int64_t>(rows, 1), db, c->stream));
    c->launches += db ? 2 : 1;
  }
  CK(c, cudaStreamSynchronize(c->stream));
  return APT_OK;
}

}  // extern "C"

// ---------------------------------------------------------------- P:163 caches
extern "C" apt_status apt_cache_sets(int64_t n, const int64_t* indptr, const int32_t* indices, const int32_t* part,
                                     int C, apt_strategy strategy, const int32_t* counts, int64_t budget,
                                     int64_t* ids_out, int64_t* n_out) {
  if (n < 1 || !counts || !ids_out || !n_out || C < 1 || C > APT_MAX_RANKS || budget < 0 ||
      ((strategy == APT_SNP || strategy == APT_DNP) && !part) || (strategy == APT_DNP && (!indptr || !indices)) ||
      strategy < APT_GDP || strategy > APT_DNP)
    return set_err(nullptr, APT_E_INVALID, "apt_cache_sets: bad arguments");
  // popularity order: count descending, id ascending (reading C1)
  std::vector<int32_t> order(n);
  for (int64_t u = 0; u < n; ++u) order[u] = int32_t(u);
  std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return counts[a] > counts[b]; });
  std::vector<uint8_t> cand(n);
  for (int r = 0; r < C; ++r) {
    if (strategy == APT_GDP || strategy == APT_NFP) {
      std::fill(cand.begin(), cand.end(), 1);
    } else {
      for (int64_t u = 0; u < n; ++u) cand[u] = part[u] == r;
      if (strategy == APT_DNP)
        for (int64_t u = 0; u < n; ++u)
          if (part[u] == r)
            for (int64_t e = indptr[u]; e < indptr[u + 1]; ++e) cand[indices[e]] = 1;
    }
    int64_t k = 0;
    for (int64_t i = 0; i < n && k < budget; ++i)
      if (cand[order[i]]) ids_out[int64_t(r) * budget + k++] = order[i];
    n_out[r] = k;
  }
  return APT_OK;
}

namespace apt {
// The store of P:163 caches: shard r = rank r's cache set (hottest first); the host tier
// holds every row (pinned, mapped, row u at u); rank r's feature map: own cache, else
// the lowest peer whose cache holds the row (NVLink), else the host.
apt_status fstore_create_p163(apt_ctx* c, const apt_graph* g, apt_strategy layout, apt_dtype dtype, int dim,
                              const float* host_feats, uint64_t feat_seed, const apt_fstore_opts* opts,
                              apt_fstore** out) {
  const int C = c->world;
  if (!opts->counts || opts->cache_budget_rows < 0 || dim <= 0 || (dtype != APT_F32 && dtype != APT_BF16))
    return set_err(c, APT_E_INVALID, "apt_fstore_create: P:163 caches need counts and a budget >= 0");
  if (layout == APT_NFP && C > 1)
    return set_err(c, APT_E_UNSUPPORTED, "apt_fstore_create: NFP keeps its column slice of every row (P:171)");
  const apt_strategy s = layout == APT_AUTO ? APT_GDP : layout;
  const int64_t B = std::min<int64_t>(opts->cache_budget_rows, g->n);
  std::vector<int64_t> ids(size_t(C) * std::max<int64_t>(B, 1)), nr(C);
  std::vector<int64_t> indptr_h;
  std::vector<int32_t> indices_h;
  if (s == APT_DNP) {
    indptr_h.resize(g->n + 1);
    indices_h.resize(g->nnz);
    CK(c, cudaMemcpy(indptr_h.data(), g->indptr, sizeof(int64_t) * (g->n + 1), cudaMemcpyDeviceToHost));
    CK(c, cudaMemcpy(indices_h.data(), g->indices, sizeof(int32_t) * g->nnz, cudaMemcpyDeviceToHost));
  }
  apt_status st = apt_cache_sets(g->n, s == APT_DNP ? indptr_h.data() : nullptr, s == APT_DNP ? indices_h.data() : nullptr,
                                 g->part_h.data(), C, s, opts->counts, B, ids.data(), nr.data());
  if (st != APT_OK) return st;
  auto* f = new apt_fstore();
  f->ctx = c;
  ctx_retain(c);
  f->g = g;
  f->layout = s;
  f->dtype = dtype == APT_BF16 ? kBF16 : kF32;
  f->dim = dim;
  f->world = C;
  f->tiered = true;
  f->p163 = true;
  f->hbm_frac = 0.0;
  const int align = dtype == APT_BF16 ? 8 : 4;
  const size_t esz = dtype == APT_BF16 ? 2 : 4;
  const int64_t pitch = round_up(dim, align);
  for (int r = 0; r < C; ++r) {
    f->col_lo[r] = 0;
    f->col_hi[r] = dim;
    f->pitch[r] = pitch;
    f->rows[r] = nr[r];
  }
  int32_t* ids_dev = f->arena.alloc<int32_t>(std::max<int64_t>(g->n, 1), false);
  auto fill = [&](void* dst, const int32_t* ids_h, int64_t n_rows) -> apt_status {
    if (n_rows <= 0) return APT_OK;
    if (host_feats) {
      std::vector<uint8_t> buf(size_t(n_rows * pitch) * esz, 0);
      for (int64_t i = 0; i < n_rows; ++i) {
        const int64_t u = ids_h ? ids_h[i] : i;
        for (int j = 0; j < dim; ++j) {
          const float v = host_feats[u * dim + j];
          if (esz == 4) {
            reinterpret_cast<float*>(buf.data())[i * pitch + j] = v;
          } else {
            uint32_t bits;
            memcpy(&bits, &v, 4);
            reinterpret_cast<uint16_t*>(buf.data())[i * pitch + j] = uint16_t((bits + 0x7FFFu + ((bits >> 16) & 1u)) >> 16);
          }
        }
      }
      CK(c, cudaMemcpyAsync(dst, buf.data(), buf.size(), cudaMemcpyDefault, c->stream));
    } else {
      const int32_t* idp = nullptr;
      if (ids_h) {
        CK(c, cudaMemcpyAsync(ids_dev, ids_h, sizeof(int32_t) * n_rows, cudaMemcpyHostToDevice, c->stream));
        idp = ids_dev;
      }
      CK(c, launch_fill_features(dst, f->dtype, pitch, 0, dim, idp, n_rows, feat_seed, c->stream));
      c->launches++;
    }
    CK(c, cudaStreamSynchronize(c->stream));
    return APT_OK;
  };
  // feature maps: holder[u] = the lowest rank caching u (-1: host only); rows inside each cache
  const int64_t n_words = ceil_div(g->n, 32);
  std::vector<int32_t> holder(g->n, -1), hrow(g->n, -1);
  std::vector<uint32_t> bm(size_t(C) * n_words, 0u), any(n_words, 0u);
  std::vector<std::vector<int32_t>> set32(C);
  for (int r = 0; r < C; ++r) {
    set32[r].resize(nr[r]);
    for (int64_t i = 0; i < nr[r]; ++i) {
      const int32_t u = int32_t(ids[size_t(r) * std::max<int64_t>(B, 1) + i]);
      set32[r][i] = u;
      bm[size_t(r) * n_words + (u >> 5)] |= 1u << (u & 31);
      any[u >> 5] |= 1u << (u & 31);
      if (holder[u] < 0) { holder[u] = r; hrow[u] = int32_t(i); }
    }
  }
  for (int r = 0; r < C; ++r) {
    if (!c->emulated && r != c->rank) continue;
    f->shard[r] = f->arena.alloc<uint8_t>(std::max<int64_t>(nr[r], 1) * pitch * int64_t(esz), true);
    if (!f->shard[r]) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "apt_fstore_create: cache"); }
    if ((st = fill(f->shard[r], set32[r].data(), nr[r])) != APT_OK) { apt_fstore_destroy(f); return st; }
  }
  f->host_rows = g->n;
  if (cudaHostAlloc(&f->host, size_t(g->n * pitch) * esz, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
    apt_fstore_destroy(f);
    return set_err(c, APT_E_OOM, "apt_fstore_create: pinned host tier of %lld rows", (long long)g->n);
  }
  if ((st = fill(f->host, nullptr, g->n)) != APT_OK) { apt_fstore_destroy(f); return st; }
  f->rows_dev = f->arena.alloc<int64_t>(C, false);
  f->cache_bm = f->arena.alloc<uint32_t>(int64_t(C) * n_words, false);
  f->any_bm = f->arena.alloc<uint32_t>(n_words, false);
  if (!f->rows_dev || !f->cache_bm || !f->any_bm) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "cache maps"); }
  CK(c, cudaMemcpyAsync(f->rows_dev, f->rows, sizeof(int64_t) * C, cudaMemcpyHostToDevice, c->stream));
  CK(c, cudaMemcpyAsync(f->cache_bm, bm.data(), sizeof(uint32_t) * bm.size(), cudaMemcpyHostToDevice, c->stream));
  CK(c, cudaMemcpyAsync(f->any_bm, any.data(), sizeof(uint32_t) * any.size(), cudaMemcpyHostToDevice, c->stream));
  for (int r = 0; r < C; ++r) {
    if (!c->emulated && r != c->rank) continue;
    std::vector<int32_t> tier(g->n), trow(g->n);
    std::vector<int32_t> own(g->n, -1);
    for (int64_t i = 0; i < nr[r]; ++i) own[set32[r][i]] = int32_t(i);
    for (int64_t u = 0; u < g->n; ++u) {
      if (own[u] >= 0) { tier[u] = r; trow[u] = own[u]; }
      else if (holder[u] >= 0) { tier[u] = holder[u]; trow[u] = hrow[u]; }
      else { tier[u] = C; trow[u] = int32_t(u); }
    }
    f->loc_map[r] = f->arena.alloc<int2>(g->n, false);
    if (!f->loc_map[r]) { apt_fstore_destroy(f); return set_err(c, APT_E_OOM, "feature map"); }
    {
      std::vector<int2> loc(g->n);
      for (int64_t u = 0; u < g->n; ++u) loc[u] = make_int2(tier[u], trow[u]);
      CK(c, cudaMemcpyAsync(f->loc_map[r], loc.data(), sizeof(int2) * g->n, cudaMemcpyHostToDevice, c->stream));
      CK(c, cudaStreamSynchronize(c->stream));
    }
    f->tier_h[r] = std::move(tier);
  }
  if (multiprocess(c)) {   // every rank maps every peer's cache (NVLink reads of peer-cached rows)
    void* tab[APT_MAX_RANKS] = {};
    apt_status s2 = share_ptr(c, f->shard[c->rank], tab, &f->peer_opened);
    if (s2 != APT_OK) { apt_fstore_destroy(f); return s2; }
    for (int r = 0; r < C; ++r) f->shard[r] = tab[r];
  }
  *out = f;
  return APT_OK;
}
}  // namespace apt
