/*
 * apt.h -- C ABI of the B200-native APT hot path.
 *
 * APT (Ma et al., "Adaptive Parallel Training for Graph Neural Networks",
 * PPoPP'25).  "P:<n>" cites line n of the paper text (reference PAPER.md).
 * The library runs the per-mini-batch sampled-subgraph step -- Philox-keyed
 * fanout sampling into CSR blocks, a gather from a feature store
 * sharded over GPUs, GraphSAGE mean aggregation and the
 * dense projection -- under the paper's four parallelisation
 * strategies GDP / NFP / SNP / DNP, plus APT's dry-run cost model
 * and strategy pick.  All kernels are hand-written sm_100a.
 *
 * Conventions (every function):
 *  - returns apt_status, never throws or aborts; the message of the last
 *    failure is apt_last_error(ctx) (valid until the next call on that ctx);
 *  - invalid arguments -> APT_E_INVALID, CUDA failure -> APT_E_CUDA (sticky:
 *    the ctx is unusable afterwards), device-side error word (bad node id,
 *    overflow) -> APT_E_DEVICE_ASSERT at the next synchronising call;
 *  - "device" pointers live on the ctx device; "host" pointers are CPU memory;
 *    the caller owns every buffer it passes in and the library copies what it
 *    keeps; objects returned through `out` are library-owned and released with
 *    the matching apt_*_destroy;
 *  - all work is stream-ordered on the ctx stream; calls documented as
 *    "syncs" block the host, all others are asynchronous;
 *  - node ids are int64 at the ABI and int32 inside (n_nodes < 2^31 checked).
 *
 * World / ranks.  A ctx hosts either one rank of a multi-process job
 * (rank >= 0; peers' symmetric buffers are attached with apt_ctx_attach_peers)
 * or all `world` ranks of an emulated job on one device (rank = -1): the same
 * kernels then address "peer" buffers that happen to live on the same GPU.
 */
#ifndef APT_H_
#define APT_H_
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  APT_OK = 0,
  APT_E_INVALID = 1,
  APT_E_OOM = 2,
  APT_E_CUDA = 3,
  APT_E_COMM = 4,
  APT_E_UNSUPPORTED = 5,
  APT_E_STATE = 6,
  APT_E_DEVICE_ASSERT = 7
} apt_status;

/* The four strategies of P:120-128 (Fig. 3) and the cost-model pick. */
typedef enum { APT_GDP = 0, APT_NFP = 1, APT_SNP = 2, APT_DNP = 3, APT_AUTO = 4 } apt_strategy;

/* Feature storage / tensor-core input type.  APT_F32: fp32 features, exact
 * fp32 CUDA-core projection (parity mode, rtol 1e-5).  APT_BF16: bf16 features,
 * Z rounded to bf16, tcgen05 bf16 projection with fp32 accumulation.          */
typedef enum { APT_F32 = 0, APT_BF16 = 1 } apt_dtype;

#define APT_MAX_LAYERS 4
#define APT_MAX_RANKS 8

typedef struct apt_ctx apt_ctx;
typedef struct apt_graph apt_graph;
typedef struct apt_fstore apt_fstore;
typedef struct apt_batch apt_batch;
typedef struct apt_trainer apt_trainer;

/* A sampled bipartite block: dst ids are the prefix of src ids;
 * CSR over local source positions.  Device pointers, borrowed from the
 * owning apt_batch (valid until it is destroyed); node ids int64 (ABI rule),
 * local positions int32.                                                    */
typedef struct {
  int64_t n_dst, n_src, n_edges;
  const int64_t* dst_ids;  /* [n_dst]   global ids (device)                 */
  const int64_t* src_ids;  /* [n_src]   global ids, dst prefix (device)     */
  const int32_t* indptr;   /* [n_dst+1] (device)                            */
  const int32_t* indices;  /* [n_edges] positions into src_ids (device)     */
} apt_block_view;

/* State the standalone first-layer forward keeps for its backward (apt_layer_fwd). */
typedef struct apt_layer_saved apt_layer_saved;

/* Model + sampler of the training task (the user's "specifics"). */
typedef struct {
  int n_layers;                        /* K                                  */
  int dims[APT_MAX_LAYERS + 1];        /* d_0 = input dim ... d_K = classes  */
  int fanouts[APT_MAX_LAYERS];         /* fanouts[l-1] for layer l (DGL)     */
  int batch;                           /* B, seeds per GPU           */
  apt_dtype dtype;
  float lr;                            /* SGD learning rate                  */
  uint64_t sample_seed;                /* Philox key of the sampler (O2)     */
  uint64_t feat_seed;                  /* synthetic features (O4)            */
  int gat_heads;                       /* 0: GraphSAGE-mean layer 1; H in {1,2,4,8}: a GAT
                                          layer 1 with H heads of dims[1]/H columns, concatenated
                                          ("GAT uses attention", [45]; G1-G4)    */
} apt_model_desc;

/* Dry-run statistics, per strategy s and rank r, summed over the
 * dry-run steps.  Bytes follow DESIGN.md §Messages.                         */
typedef struct {
  int world;
  int64_t steps;
  int64_t n_d[4][APT_MAX_RANKS];             /* layer-1 destinations N_d          */
  int64_t n_vs[APT_MAX_RANKS];               /* SNP virtual nodes          */
  int64_t n_vd[APT_MAX_RANKS];               /* DNP virtual nodes          */
  int64_t rows_local[4][APT_MAX_RANKS];      /* unique feature rows read locally   */
  int64_t rows_peer[4][APT_MAX_RANKS];       /* ... read from a peer GPU (NVLink)  */
  int64_t feat_bytes_local[4][APT_MAX_RANKS];
  int64_t feat_bytes_peer[4][APT_MAX_RANKS];
  int64_t graph_bytes[4][APT_MAX_RANKS];     /* Shuffle: computation graph received */
  int64_t hidden_bytes_fwd[4][APT_MAX_RANKS];/* Reshuffle fwd: hidden received     */
  int64_t hidden_bytes_bwd[4][APT_MAX_RANKS];/* Reshuffle bwd: gradients received  */
  int64_t n_calls[4][APT_MAX_RANKS];         /* exchange operators per step        */
  double t_build_s[4][APT_MAX_RANKS];        /* measured T_build           */
  double t_train_s;                          /* measured common T_train (GDP)      */
  int64_t rows_host[4][APT_MAX_RANKS];       /* unique rows read from the host tier */
  int64_t feat_bytes_host[4][APT_MAX_RANKS];
  /* GAT layer 1 (gat_heads > 0): the extra exchange attention costs NFP and SNP
   * (Fig. 10 / P:344).  NFP: the partial score and dalpha sums,
   * reduced into and read back from every other requester (4 passes x H x 4 B per
   * edge); SNP: the softmax state (m, S) with every partial and (t, L) with every
   * gradient (2H x 4 B each way per virtual node) and, per item an owner
   * computes, the destination's own feature row (attn_feat_bytes, NVLink).
   * GDP and DNP: 0 ("each destination node has a complete view").      */
  int gat_heads;
  int64_t attn_bytes[4][APT_MAX_RANKS];
  int64_t attn_feat_bytes[4][APT_MAX_RANKS];
  /* Reading R1: owners re-sample the rows requesters route to them with the same Philox
   * key; that time (measured layer-1 sampling cost per row x rows re-sampled) is
   * included in t_build_s and reported here.                                        */
  double t_resample_s[4][APT_MAX_RANKS];
  double t_dryrun_s;                         /* host wall time of the whole dry run */
} apt_plan_stats;

/* Operator slots of the bandwidth profile ("trials").          */
enum {
  APT_OP_LOCAL_GATHER = 0, APT_OP_PEER_PULL = 1, APT_OP_PEER_PUSH = 2, APT_OP_ALLTOALLV = 3,
  APT_OP_ALLGATHER = 4, APT_OP_REDUCE_SCATTER = 5, APT_OP_ALLREDUCE = 6, APT_OP_HOST_GATHER = 7
};
typedef struct {
  int world;
  double alpha_s[8];     /* per-call latency of each operator (reading Z23) */
  double beta_Bps[8];    /* bytes per second of each operator                */
  int measured[8];       /* 1: timed by apt_profile_links on this process;
                            0: the pool's measured NVLink reference (no peer GPU) */
} apt_bw_profile;

/* All-gather used to bootstrap a job of one process per GPU: every rank passes
 * `bytes` bytes in `send`; on return `recv` holds world*bytes bytes, rank p's
 * block at offset p*bytes.  Returns 0 on success.  (The Python binding supplies
 * one built on torch.distributed.)  Used only while creating objects, never on
 * the step path.                                                            */
typedef int (*apt_allgather_fn)(const void* send, void* recv, size_t bytes, void* user);

/* ---------------------------------------------------------------- context */
/* rank >= 0: one rank of `world`; rank == -1: all `world` ranks emulated on
 * `device`.  cuda_stream may be NULL (library-created stream).              */
apt_status apt_ctx_create(int rank, int world, int device, void* cuda_stream, apt_ctx** out);
apt_status apt_ctx_destroy(apt_ctx* ctx);
const char* apt_last_error(const apt_ctx* ctx);
/* Multi-process job (rank >= 0, world > 1): install the bootstrap all-gather.
 * Collective.  Sets up the device barrier (peer-mapped flag arrays); objects
 * created afterwards map their peers' buffers through CUDA IPC.              */
apt_status apt_ctx_set_exchange(apt_ctx* ctx, apt_allgather_fn fn, void* user);
/* Host-only check of an exchange function's protocol (no GPU used). Collective. */
apt_status apt_exchange_selftest(int rank, int world, apt_allgather_fn fn, void* user);
/* Syncs: waits for the ctx stream and reports device-side error words.      */
apt_status apt_ctx_sync(apt_ctx* ctx);
/* Copy helper for tests/bindings: kind 0 = D2H, 1 = H2D, 2 = D2D. Syncs.   */
apt_status apt_memcpy(apt_ctx* ctx, void* dst, const void* src, size_t bytes, int kind);
/* Number of kernels this ctx launched so far (evidence for gpu_launches).   */
int64_t apt_ctx_launches(const apt_ctx* ctx);

/* ------------------------------------------------------------------ graph */
/* Copies a symmetric CSR (host) into HBM, replicated per device (P:186 keeps
 * topology replicated).  part: host int32[n] owner of every node (edge-cut
 * partition); NULL => range partition floor(u*world/n).  Syncs.      */
apt_status apt_graph_load(apt_ctx* ctx, int64_t n_nodes, int64_t nnz, const int64_t* indptr,
                          const int32_t* indices, const int32_t* part, apt_graph** out);
apt_status apt_graph_destroy(apt_graph* g);

/* ------------------------------------------------------------ feature store */
/* Unified feature store laid out for `layout`:
 * GDP/SNP/DNP: rows sharded by part (rank r holds its partition's rows);
 * NFP: columns sharded, rank c holds columns [c*d/C, (c+1)*d/C) of all rows.
 * host_feats: host fp32 [n x dim] or NULL => synthetic O4 features from
 * feat_seed generated on the device.  Rows padded to 16 bytes.  Syncs.      */
apt_status apt_fstore_create(apt_ctx* ctx, const apt_graph* g, apt_strategy layout, apt_dtype dtype,
                             int dim, const float* host_feats, uint64_t feat_seed, apt_fstore** out);
apt_status apt_fstore_destroy(apt_fstore* f);

/* Tiers of the unified feature store. */
typedef struct {
  double hbm_frac;          /* fraction of every partition's rows kept in its owner's HBM (1.0: all); the
                               rest form the host tier (pinned, mapped; read over PCIe / C2C)          */
  int64_t cache_rows;       /* excess cache: rows replicated into every GPU's spare HBM */
  const int64_t* hot_ids;   /* host, >= cache_rows candidate ids, hottest first (apt_hot_rows)        */
  /* P:163 "Cache configuration" (cache_rule = APT_CACHE_P163; hbm_frac / cache_rows unused):
   * every GPU's HBM holds only its cache set -- the cache_budget_rows most popular nodes
   * under the store layout's strategy rule (apt_cache_sets, from the dry-run counts) --
   * and the host tier holds every row; a row is read from the own cache, else from a
   * peer GPU's cache over NVLink, else from the host (the feature map of P:241-247).   */
  int cache_rule;
  const int32_t* counts;    /* host int32[n]: access frequencies (apt_access_counts)                   */
  int64_t cache_budget_rows;
} apt_fstore_opts;
enum { APT_CACHE_NONE = 0, APT_CACHE_P163 = 1 };
/* The per-GPU cache sets of P:163: GDP / NFP the most popular nodes of the graph, SNP
 * of the GPU's partition, DNP of its partition and their 1-hop neighbours; popularity =
 * counts descending, ties by ascending id; at most `budget` ids per GPU.  Host CSR
 * (symmetric), part host int32[n]; ids_out host int64 [C x budget] (rank r's ids,
 * hottest first, at ids_out + r * budget), n_out host int64 [C].  Host only.           */
apt_status apt_cache_sets(int64_t n, const int64_t* indptr, const int32_t* indices, const int32_t* part, int C,
                          apt_strategy strategy, const int32_t* counts, int64_t budget, int64_t* ids_out,
                          int64_t* n_out);
/* apt_fstore_create with tiers (opts NULL: everything in HBM).  Row-sharded
 * layouts only (NFP: APT_E_UNSUPPORTED: NFP keeps its 1/C column slice of every row,
 * with that much memory it reads nothing from the host).  Kernels see one view per rank: own
 * HBM rows, NVLink peer rows, host rows, own cached rows.  Syncs.            */
apt_status apt_fstore_create_tiered(apt_ctx* ctx, const apt_graph* g, apt_strategy layout, apt_dtype dtype,
                                    int dim, const float* host_feats, uint64_t feat_seed, const apt_fstore_opts* opts,
                                    apt_fstore** out);

/* -------------------------------------------------------------- partition */
/* Edge-cut partitioners of APT's Prepare stage for SNP / DNP ("edge-cut (e.g.,
 * METIS)"; Fig. 11 / P:346 quality ablation):
 *   APT_PART_RANGE   floor(u C / n)       (the generator's planted partition);
 *   APT_PART_RANDOM  Philox(seed; u) mod C (Fig. 11's random partition);
 *   APT_PART_LDG     linear deterministic greedy streaming (reading R10): nodes in
 *                    ascending id, u -> argmax over p with size_p < cap of
 *                    |N(u) in P_p| * (cap - size_p), ties to the smaller size_p then
 *                    the smaller p, cap = ceil(1.05 n / C).
 * Host CSR (symmetric), writes part[n] (host int32); *cut_edges (may be NULL) = CSR
 * entries (u, v) with part[u] != part[v].  Host only, no ctx.                   */
enum { APT_PART_RANGE = 0, APT_PART_RANDOM = 1, APT_PART_LDG = 2 };
apt_status apt_partition(int64_t n, int64_t nnz, const int64_t* indptr, const int32_t* indices, int C, int method,
                         uint64_t seed, int32_t* part, int64_t* cut_edges);

/* ---------------------------------------------------------------- sampling */
/* K-hop node-wise sampling of seeds_dev (device int64[n_seeds]) with
 * fanouts (host, fanouts[l-1] for layer l, 1..256), Philox key rng_seed and
 * step id `step` (reading O2).  Builds hop-h blocks h = 0..K-1 (layer l's
 * block is hop K-l).  Syncs once at the end (block sizes).                  */
apt_status apt_sample(apt_ctx* ctx, const apt_graph* g, const int64_t* seeds_dev, int64_t n_seeds,
                      const int32_t* fanouts, int n_layers, uint64_t rng_seed, uint64_t step,
                      apt_batch** out);
apt_status apt_batch_block(const apt_batch* b, int hop, apt_block_view* out);
apt_status apt_batch_destroy(apt_batch* b);
/* A ctx hosting several ranks (rank = -1 emulation) runs the layer API on one batch
 * per hosted rank: per_rank[i] is hosted rank i's batch (same graph, K, fanouts,
 * rng_seed and step).  The group borrows the batches: keep them alive until the group
 * is destroyed (apt_batch_destroy).  apt_batch_block on a group -> APT_E_INVALID.    */
apt_status apt_batch_group(apt_ctx* ctx, const apt_batch* const* per_rank, int n, apt_batch** out);

/* ------------------------------------------------------------ single ops */
/* Gather rows of ids_dev (device int64[n], node ids) from this rank's view of the
 * store (own shard, NVLink peers, host tier, cache) into out_dev
 * (device, rows of the store's padded pitch, store dtype).  An id outside
 * [0, n_nodes) -> APT_E_DEVICE_ASSERT at the next sync (its row is node 0's).  */
apt_status apt_gather(apt_ctx* ctx, const apt_fstore* f, const int64_t* ids_dev, int64_t n, void* out_dev);
/* Segmented mean (O5): z[v] = mean_{e in row v} x[indices[e]].  x_src device
 * [n_src x x_pitch] of dtype; z_dst device fp32 [n_dst x z_pitch].          */
apt_status apt_aggregate(apt_ctx* ctx, const apt_block_view* blk, const void* x_src, apt_dtype dtype,
                         int dim, int64_t x_pitch, float* z_dst, int64_t z_pitch);
/* Backward of the mean: dx[indices[e]] += dz[v]/deg(v) (accumulates).       */
apt_status apt_aggregate_bwd(apt_ctx* ctx, const apt_block_view* blk, const float* dz, int dim, int64_t dz_pitch,
                             float* dx_src, int64_t dx_pitch);
/* Projection Y = Z W^T + b (+ReLU) (Eq. 1) on the tensor cores.  dtype
 * APT_BF16: Z is bf16 [M x z_pitch], W rounded to bf16, kind::f16 with fp32
 * accumulation (N, K <= 256: the row-tile kernel with W resident; wider: the general
 * kernel, N tiled and K streamed); APT_F32: Z fp32, 3xTF32 on kind::tf32 (each product
 * carried to ~2^-21, reading P1), falling back to exact fp32 CUDA cores when a pitch is
 * not a 16-byte multiple.  W device fp32 [N x K]; Y device fp32 [M x y_pitch].  Syncs. */
apt_status apt_project(apt_ctx* ctx, const void* Z, int64_t z_pitch, apt_dtype dtype, const float* W,
                       const float* bias, int64_t M, int N, int K, int relu, float* Y, int64_t y_pitch);

/* Weight gradient of the projection (S11; reading O5): dW[o][i] += sum_r
 * G[r][o] Z[r][i] and db[o] += sum_r G[r][o] over rows r < rows (accumulates
 * into dW [d_out x d_in] and db [d_out], device fp32; db may be NULL).  G device
 * fp32 [rows x g_pitch]; Z device [rows x z_pitch] of dtype.  APT_BF16: G is
 * rounded to bf16 and the contraction runs on tcgen05 kind::f16 (any d_out, d_in);
 * APT_F32: 3xTF32 on kind::tf32 (CUDA cores if a pitch is not a 16-byte multiple).
 * Syncs.                                                                    */
apt_status apt_weight_grad(apt_ctx* ctx, const float* G, int64_t g_pitch, const void* Z, int64_t z_pitch,
                           apt_dtype dtype, int64_t rows, int d_out, int d_in, float* dW, float* db);

/* ------------------------------------------------------------------ trainer */
/* The per-mini-batch step (P:110 sampling -> loading -> training) under one
 * strategy, for every rank hosted by ctx.  labels: host int32[n_nodes].      */
apt_status apt_trainer_create(apt_ctx* ctx, const apt_graph* g, const apt_fstore* f, const apt_model_desc* m,
                              apt_strategy s, const int32_t* labels, apt_trainer** out);
apt_status apt_trainer_destroy(apt_trainer* t);
/* Host fp32 W [d_out x d_in] row-major and b [d_out] of layer l (1..K); every rank. */
apt_status apt_trainer_set_params(apt_trainer* t, int layer, const float* W, const float* b);
apt_status apt_trainer_get_params(apt_trainer* t, int rank, int layer, float* W, float* b);
/* GAT layer 1 (gat_heads > 0) attention vectors, host fp32 [dims[1]] each, head h at
 * [h*F, (h+1)*F): e_vu^h = LeakyReLU_0.2(a_src^h . (W x_u)^h + a_dst^h . (W x_v)^h)
 * (GAT [45]; reading G1).  Replicated on every rank; updated by SGD.
 * APT_E_STATE on a SAGE layer 1.  Syncs.                                     */
apt_status apt_trainer_set_attention(apt_trainer* t, const float* a_src, const float* a_dst);
apt_status apt_trainer_get_attention(apt_trainer* t, int rank, float* a_src, float* a_dst);
/* Epoch permutation of the train set (O1): host int64[n_train] ascending.   */
apt_status apt_trainer_set_epoch(apt_trainer* t, const int64_t* train, int64_t n_train, uint64_t epoch);
int64_t apt_trainer_steps_per_epoch(const apt_trainer* t);
/* One training step: seeds of step `step` of the epoch, sampling, layer-1
 * strategy forward (Permute/Shuffle/Execute/Reshuffle), upper
 * layers, CE loss, backward, gradient all-reduce, SGD if update != 0.  Async. */
apt_status apt_trainer_step(apt_trainer* t, int64_t step, int update);
/* Same, but the global batch comes from host memory (pinned for overlap),
 * copied in on the stream, and the loss is copied back: the end-to-end call.
 * Syncs.                                                                    */
apt_status apt_trainer_step_host(apt_trainer* t, const int64_t* gbatch_host, int64_t n_global, int64_t step,
                                 int update, float* loss_host);
/* Pipelined end-to-end call: submit the NEXT global batch (host int64 ids, step id
 * next_step) and run the step of the batch the previous call submitted, returning
 * its loss in *loss_prev (*had_step = 1).  The next batch's H2D copy and sampling
 * overlap the step (second sample set, sampling stream).  The first call only
 * primes (*had_step = 0).  Syncs.                                           */
apt_status apt_trainer_step_host_pipelined(apt_trainer* t, const int64_t* next_batch, int64_t n_next,
                                           int64_t next_step, int update, float* loss_prev, int* had_step);
/* The same pipelined end-to-end call without waiting for the step it launches: it
 * writes the next batch into pinned staging, launches this call's step (H2D of the next
 * batch, the step, D2H of its loss) and then waits only for the step the PREVIOUS call
 * launched, returning that step's loss (*had_step = 0 on the first two calls) -- the
 * device always has the next step queued while the host prepares the next call.  Use
 * apt_trainer_loss (syncs) for the last step's loss.  Device error words surface at the
 * next synchronising call.                                                          */
apt_status apt_trainer_step_host_async(apt_trainer* t, const int64_t* next_batch, int64_t n_next, int64_t next_step,
                                       int update, float* loss_prev, int* had_step);
/* Loss of the last step (sum over ranks).  Syncs.                           */
apt_status apt_trainer_loss(apt_trainer* t, float* loss);
/* Record/replay the device part of apt_trainer_step as a CUDA graph.        */
apt_status apt_trainer_use_graph(apt_trainer* t, int enable);
/* Pipelining (default on): while step t computes, step t+1's mini-batch is
 * sampled into a second buffer set on a separate stream (SURVEY §8(f) NEXT #4,
 * P:299 "sampling" overlapped).  Results are identical with it off.          */
apt_status apt_trainer_set_pipeline(apt_trainer* t, int enable);

/* The first GNN layer alone -- the layer APT parallelises (the
 * sampler and the upper layers are the user's black boxes).
 *
 * apt_layer_fwd: h1 = ReLU(mean-aggregate(x) W^T + bias) of the layer-1 block of
 *   `batch` (hop K-1 of apt_sample's output; Eq. 1 with W after the mean, Z8; ReLU
 *   because layer 1 is a hidden layer, Z9) under `strategy`'s Permute / Shuffle /
 *   Execute / Reshuffle.  Collective for a multi-process job.
 *   batch: this rank's batch, or for an emulated ctx an apt_batch_group of every
 *   hosted rank's batch.  fstore: laid out for the strategy (NFP: column-sharded),
 *   its dtype = `dtype`.  W: device fp32 [d_out x d] row-major, bias: device fp32
 *   [d_out] (replicated: every rank passes the same values).  h1_out: device fp32
 *   [rows x d_out], the hosted ranks' layer-1 destinations concatenated in rank
 *   order (rows = sum of n_dst of each batch's layer-1 block); bf16 mode writes the
 *   stored bf16 activation (R11) widened to fp32.  *saved: library-owned, needed by
 *   apt_layer_bwd, released with apt_layer_saved_destroy.  Async (one host sync while
 *   staging the blocks).
 * apt_layer_bwd: dh1 = device fp32 dL/dh1 in h1_out's layout; computes g = dh1 *
 *   ReLU'(pre) and dW = g^T Z (owners' partial sums, NFP column-owned slices), db = g^T 1
 *   at the requester (R3), all-reduced over the ranks.  dW: device fp32
 *   [d_out x d]: the full gradient (NFP: the hosted ranks' column slices, other columns
 *   untouched); dbias: device fp32 [d_out].  Collective; async.                      */
apt_status apt_layer_fwd(apt_ctx* ctx, apt_strategy strategy, const apt_batch* batch, const apt_fstore* fstore,
                         const float* W, const float* bias, int d_out, apt_dtype dtype, float* h1_out,
                         apt_layer_saved** saved);
apt_status apt_layer_bwd(apt_ctx* ctx, apt_layer_saved* saved, const float* dh1, float* dW, float* dbias);
apt_status apt_layer_saved_destroy(apt_layer_saved* saved);

/* The same first layer bound to a trainer (its model, epoch and strategy):
 * apt_trainer_layer_fwd samples step `step` of the epoch for every hosted rank and runs
 * the layer-1 forward (SAGE or GAT); h^1 is read with apt_trainer_read(H, layer 1).
 * apt_trainer_layer_bwd: dh1[i] = device fp32 dL/dh^1 of hosted rank i (rows = its
 * layer-1 destinations, `pitch` floats apart); dW^1, db^1 (GAT: also da_src, da_dst)
 * of the strategy, all-reduced (NFP: column-owned slices).  Async.                   */
apt_status apt_trainer_layer_fwd(apt_trainer* t, int64_t step);
apt_status apt_trainer_layer_bwd(apt_trainer* t, const float* const* dh1, int64_t pitch);

/* Readouts for tests (syncs).  what: 0 seeds, 1 layer-l dst ids, 2 Z_l (fp32),
 * 3 H_l (post-activation / logits), 4 dW_l, 5 db_l, 6 G_l (dL/dpre),
 * 7 (GAT layer 1) the attention gradients [da_src | da_dst] (1 x 2*dims[1]).
 * Copies min(cap, rows*cols) values (int32 for ids, fp32 otherwise).         */
apt_status apt_trainer_read(apt_trainer* t, int rank, int what, int layer, void* host, int64_t cap,
                            int64_t* rows, int* cols);
/* Per-phase device time of the last step in ms (CUDA events), n <= 16:
 * 0 seeds+sampling, 1 layer-1 fwd, 2 upper fwd + loss, 3 backward, 4 allreduce+SGD,
 * 5 dominant kernel (layer-1 gather+aggregate).  Syncs.                      */
apt_status apt_trainer_phase_ms(apt_trainer* t, double* ms, int n);
/* Algorithmic bytes of the last step's layer-1 gather+aggregate. Syncs. */
apt_status apt_trainer_agg_bytes(apt_trainer* t, double* bytes);

/* ------------------------------------------------------------------ planner */
/* Dry-run: samples `n_steps` steps of the current epoch,
 * runs Permute+Shuffle of every strategy on the shared samples (no feature
 * loading, no training), counts volumes and times T_build.  Syncs.          */
apt_status apt_dryrun(apt_trainer* t, int64_t n_steps, apt_plan_stats* out);
/* Node access frequencies (Table 3; reading R12): counts_host[u]
 * (host int32 [n], caller-owned, overwritten) = number of (step, requester)
 * pairs of the first n_steps global steps of the current epoch (GDP seed split)
 * whose layer-1 block has u as a source, i.e. how often u's input row is loaded.
 * Same sampler as the step (bit-identical blocks).  Syncs.                   */
apt_status apt_access_counts(apt_trainer* t, int64_t n_steps, int32_t* counts_host);
/* Hot list of the excess cache: the k ids with the largest
 * counts[] (host int32 [n]), descending, ties by ascending id, into ids_out
 * (host int64 [k], caller-owned).  Pure host arithmetic; APT_E_INVALID if
 * k > n or a pointer is NULL.                                               */
apt_status apt_hot_rows(const int32_t* counts, int64_t n, int64_t k, int64_t* ids_out);
/* Bandwidth trials of the exchange operators: each operator this
 * process can run is timed at two message sizes and fitted to alpha + bytes/beta
 * (local HBM row gather, pinned-host read); NVLink operators take the pool's
 * measured references when no peer GPU is attached (measured[op] = 0).  Syncs. */
apt_status apt_profile_links(apt_ctx* ctx, apt_bw_profile* out);
/* Eq. 2 without the common T_train: pred_s[s] = max over ranks of
 * T_build + T_load + T_shuffle; *pick = argmin.  Pure host arithmetic.      */
apt_status apt_select_strategy(const apt_plan_stats* st, const apt_bw_profile* bw, apt_strategy* pick,
                               double pred_s[4]);

/* Self-test of the mean's division (reading O5): the number of operands for which
 * the reciprocal-based correctly-rounded division differs bitwise from IEEE
 * x / d over every O4 mean (x = m/64, |m| <= 2^17, d = 1..256) and random normal
 * numerators; 0 expected, < 0 on a CUDA failure.  Uses the current device.      */
int64_t apt_selftest_div(void);

/* Self-test of the epoch permutation's sort (S1, reading O1; sort.cu): n (key, value)
 * pairs with Philox keys masked to key_bits bits (equal keys when key_bits is small),
 * values 0..n-1, sorted on the device by the library's stable LSD radix sort; returns
 * the number of positions that differ from a host std::stable_sort, < 0 on failure.
 * Uses the current device; syncs.                                                    */
int64_t apt_selftest_sort(int64_t n, uint64_t seed, int key_bits);

/* Self-test of the general tensor-core contraction (gemm_tc_gen.cu): C = A B + bias for
 * fp32 (3xTF32, f32 = 1) or bf16 operands, A / B K-major or M/N-major, M x N x K, split-K
 * accumulating when `accumulate`; returns max |C - ref| / (sum_k |A||B| + |bias|) against
 * an fp64 host product, < 0 on failure.  Uses the current device; syncs.             */
double apt_selftest_gemm(int f32, int a_mn, int b_mn, int64_t M, int N, int64_t K, int accumulate);

#ifdef __cplusplus
}
#endif
#endif /* APT_H_ */
