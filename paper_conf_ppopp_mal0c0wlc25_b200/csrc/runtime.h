// runtime.h -- internal host-side structures behind the C ABI (include/apt.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/apt.h"
#include "kernels.h"

namespace apt {

// Device allocation owned by one library object.
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
};

struct Arena {
  std::vector<DevBuf> bufs;
  size_t total = 0;
  ~Arena() { release(); }
  void release() {
    for (auto& b : bufs) cudaFree(b.p);
    bufs.clear();
    total = 0;
  }
  template <typename T>
  T* alloc(int64_t n, bool zero = true) {
    void* p = nullptr;
    size_t bytes = size_t(std::max<int64_t>(n, 1)) * sizeof(T);
    bytes = (bytes + 255) & ~size_t(255);
    if (cudaMalloc(&p, bytes) != cudaSuccess) return nullptr;
    // cudaMemset runs on the legacy stream, which does not order against the ctx's
    // non-blocking stream: wait for it, or a later kernel's output could be zeroed
    if (zero && (cudaMemset(p, 0, bytes) != cudaSuccess || cudaStreamSynchronize(cudaStreamLegacy) != cudaSuccess)) {
      cudaFree(p);
      return nullptr;
    }
    bufs.push_back({p, bytes});
    total += bytes;
    return static_cast<T*>(p);
  }
};

// Child objects keep their ctx alive: a ctx destroyed before them is released by
// the last child (any destruction order is safe, e.g. at interpreter exit).
void ctx_retain(apt_ctx* c);
void ctx_release(apt_ctx* c);

// comm.cu: one process per GPU
bool multiprocess(const apt_ctx* c);
apt_status allgather(apt_ctx* c, const void* send, void* recv, size_t bytes);
apt_status share_ptr(apt_ctx* c, void* local, void** tab, std::vector<void*>* opened);
void close_peers(std::vector<void*>& opened);
apt_status device_barrier(apt_ctx* c);
// Multi-process: an exporter may free a buffer only after every importer closed its
// mapping (CUDA IPC rule), so objects hand their buffers to the ctx, which frees them
// at its (collective) destruction behind a host barrier.
void defer_exported(apt_ctx* c, Arena& a);

}  // namespace apt

struct apt_ctx {
  int rank = 0;          // first hosted rank
  int world = 1;
  int n_local = 1;       // ranks hosted by this ctx
  bool emulated = false;
  int device = 0;
  int sm_count = 148;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  cudaStream_t side = nullptr;           // forked branch of a step (weight gradients off the critical path)
  cudaStream_t samp = nullptr;           // sampling of the next step (pipelined trainer)
  cudaStream_t samp2 = nullptr;          // its block transposes, off the sampling chain (APT_BG_CSC_FORK)
  cudaEvent_t ev_sfork = nullptr, ev_sjoin = nullptr;
  cudaStream_t tap = nullptr;            // captured graphs: timing events hang off the chain here
  cudaEvent_t ev_tap = nullptr, ev_tapj = nullptr;
  cudaEvent_t ev_pfork = nullptr, ev_pjoin = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_csc = nullptr;
  bool broken = false;
  std::string err;
  int64_t launches = 0;
  int children = 0;      // live graphs / stores / batches / trainers created on this ctx
  apt_allgather_fn exchange = nullptr;   // multi-process bootstrap (apt_ctx_set_exchange)
  void* exchange_user = nullptr;
  uint64_t* bar_flags = nullptr;         // [APT_MAX_RANKS] arrival slots + epoch (device barrier)
  uint64_t** bar_tab = nullptr;          // every rank's bar_flags (peer-mapped)
  std::vector<void*> peer_opened;        // IPC mappings to close
  std::vector<apt::DevBuf> deferred;     // exported buffers of destroyed objects: freed only at
                                         // ctx destroy, after every peer has closed its mapping
  bool zombie = false;   // apt_ctx_destroy called while children were alive
  uint32_t* dev_err = nullptr;   // device error word
  int32_t* scratch = nullptr;    // small device ints for single-op calls
  apt::Arena arena;
};

struct apt_graph {
  apt_ctx* ctx = nullptr;
  int64_t n = 0, nnz = 0;
  int64_t* indptr = nullptr;     // device
  int32_t* indices = nullptr;    // device
  int32_t* part = nullptr;       // device owner of every node
  int32_t* lrow = nullptr;       // device row inside the owner's shard
  int2* loc = nullptr;           // device (part, lrow) of every node: the feature view's one 8-B load
  std::vector<int32_t> part_h;   // host copy
  std::vector<int64_t> shard_rows;   // rows per rank
  int world = 1;
  apt::Arena arena;
};

struct apt_fstore {
  apt_ctx* ctx = nullptr;
  const apt_graph* g = nullptr;
  apt_strategy layout = APT_GDP;
  apt::DType dtype = apt::kF32;
  int dim = 0;
  int world = 1;
  // per rank shard
  void* shard[APT_MAX_RANKS] = {};
  int64_t pitch[APT_MAX_RANKS] = {};   // elements per row
  int col_lo[APT_MAX_RANKS] = {};
  int col_hi[APT_MAX_RANKS] = {};
  int64_t rows[APT_MAX_RANKS] = {};      // rows of each shard held in HBM
  // tiers (apt_fstore_opts): host tier + per-rank hot-row caches, and the per-rank maps
  bool tiered = false;
  double hbm_frac = 1.0;
  int64_t host_rows = 0;
  void* host = nullptr;                  // pinned, mapped: rows beyond every shard's HBM budget
  int64_t cache_rows[APT_MAX_RANKS] = {};
  void* cache[APT_MAX_RANKS] = {};       // replicated hot rows (hosted ranks)
  int2* loc_map[APT_MAX_RANKS] = {};     // device [n] per hosted rank: (tier, row) of every node
  std::vector<int32_t> tier_h[APT_MAX_RANKS];   // host copies (tests)
  // for the dry-run's tier classification of every rank's reads (all ranks, any process):
  // u is local to r iff cached by r or (part[u] == r and lrow[u] < rows[r]); host iff
  // lrow[u] >= rows[part[u]] and not cached by r
  int64_t* rows_dev = nullptr;           // [C] HBM rows per shard
  uint32_t* cache_bm = nullptr;          // [C x ceil(n/32)] cached-by-rank bitmaps (null: no caches)
  bool p163 = false;                     // APT_CACHE_P163: shards are the per-GPU cache sets
  uint32_t* any_bm = nullptr;            // ... cached by some rank (NVLink-readable)
  std::vector<void*> peer_opened;   // IPC-mapped peer shards (multi-process)
  apt::Arena arena;
  ~apt_fstore() {
    apt::close_peers(peer_opened);
    apt::defer_exported(ctx, arena);
    if (host) cudaFreeHost(host);
  }
};

struct apt_batch {
  apt_ctx* ctx = nullptr;
  const apt_graph* g = nullptr;
  int K = 0;
  uint64_t rng_seed = 0, step = 0;             // the sampler's Philox key and step id (O2)
  int fanouts[APT_MAX_LAYERS] = {};            // fanouts[l-1] of layer l
  int64_t n_dst[APT_MAX_LAYERS] = {}, n_src[APT_MAX_LAYERS] = {}, n_edges[APT_MAX_LAYERS] = {};
  int32_t* dst[APT_MAX_LAYERS] = {};
  int32_t* src[APT_MAX_LAYERS] = {};
  int32_t* indptr[APT_MAX_LAYERS] = {};
  int32_t* indices[APT_MAX_LAYERS] = {};
  int32_t* cnt[APT_MAX_LAYERS] = {};           // the sampler's ELL form of every hop (fixed stride k)
  int32_t* nbr[APT_MAX_LAYERS] = {};
  int32_t* counts = nullptr;                   // device: [0] n_seeds, [1 + 2h] n_src(h), [2 + 2h] n_edges(h)
  int64_t* dst64[APT_MAX_LAYERS] = {};         // int64 copies of the ids for apt_block_view (ABI rule)
  int64_t* src64[APT_MAX_LAYERS] = {};
  std::vector<const apt_batch*> members;       // apt_batch_group: one borrowed batch per hosted rank
  apt::Arena arena;
};
