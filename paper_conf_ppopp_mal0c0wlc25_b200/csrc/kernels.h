// kernels.h -- launcher declarations for the sm_100a kernels (internal, C++).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace apt {

// Workspace granularity of the single-pass scans (sample.cu): one status word pair per
// tile; the scans' tile (kScanThreads * kScanItems) must be a multiple of it.
constexpr int kScanWsTile = 512;

// ---------------------------------------------------------------- sample.cu
struct SampleArgs {
  const int64_t* indptr;
  const int32_t* indices;
  const int32_t* frontier;
  const int32_t* n_frontier;   // device count
  int64_t max_frontier;        // grid upper bound
  int k;
  uint2 key;
  const uint64_t* step;        // device step id
  int hop;
  int32_t* cnt;                // [max_frontier]
  int32_t* nbr;                // [max_frontier * k] global ids, fixed stride k
  int64_t grid_cap;            // max blocks (0: default) -- background sampling uses few SMs
};
cudaError_t launch_sample(const SampleArgs& a, cudaStream_t st);

struct CompactArgs {
  const int32_t* dst;          // frontier (dst ids)
  const int32_t* n_dst;
  int64_t max_dst;
  const int32_t* cnt;
  const int32_t* nbr;
  int k;
  uint32_t* dst_bm;            // [n_words], zero on entry and exit
  uint32_t* new_bm;            // [n_words], zero on entry and exit
  int64_t n_words;
  int32_t* pos;                // [n_nodes] scratch global->local map
  int32_t* src;                // [max_src]
  int32_t* n_src;
  int32_t* indptr;             // [max_dst + 1]
  int32_t* indices;            // [max_dst * k]
  int32_t* n_edges;
  int32_t* partials;           // scan workspace (>= 2 * n_words / kScanWsTile + 8)
  int32_t* partials2;          // scan workspace (>= 2 * max_dst / kScanWsTile + 8)
  int64_t grid_cap;            // max blocks of the grid-stride kernels (0: default)
  // optional: the block transpose's in-degree count, done while the indices are mapped
  // (csc_cnt zero on entry), and the reset of its scan's status words / ticket
  int32_t* csc_cnt; uint64_t* csc_st; int csc_nb; int32_t* csc_ticket;
};
cudaError_t launch_compact(const CompactArgs& a, cudaStream_t st);
int scan_tiles(int64_t max_n);   // status pairs of a look-back scan over max_n items

struct SeedArgs {
  const int32_t* perm;
  int64_t n_train;
  const uint64_t* step;
  int64_t steps_per_epoch;
  int world, rank, batch, by_part;
  const int32_t* part;
  int32_t* seeds;
  int32_t* n_seeds;
  int32_t* n_global;
  const int32_t* n_dev;        // if set: perm is one global batch of *n_dev ids (host-batch path)
};
cudaError_t launch_select_seeds(const SeedArgs& a, cudaStream_t st);
// layer_api.cu: int32 <-> int64 node ids at the ABI.
cudaError_t launch_widen_ids(const int32_t* a, int64_t n, int64_t* b, cudaStream_t st);
cudaError_t launch_narrow_ids(const int64_t* a, int64_t n, int64_t n_nodes, int32_t* b, uint32_t* err, cudaStream_t st);
// sort.cu: stable LSD radix sort of (uint64 key, int32 value) pairs in place (S1, O1).
size_t radix_sort_pairs_scratch(int64_t n);
cudaError_t launch_radix_sort_pairs(uint64_t* keys, int32_t* vals, int64_t n, void* scratch, cudaStream_t st);
cudaError_t launch_perm_keys(const int32_t* train, int64_t n, uint64_t seed, uint64_t epoch, uint64_t* keys,
                             cudaStream_t st);

// ------------------------------------------------------------------ agg.cu
enum DType : int { kF32 = 0, kBF16 = 1 };

// Feature store view used by the fused gather+mean kernel (S6+S7).
// Unified feature store as seen by one rank: tier t of node u is
// part[u]: 0..C-1 = that rank's HBM shard (local or NVLink peer), C = the host tier
// (pinned, mapped), C+1 = this rank's cache of replicated hot rows.
struct FeatView {
  const void* base[10];        // per-tier base (local / NVLink peer / mapped host / own cache)
  const int2* loc;             // (tier, row inside the tier) of node u: ONE 8-byte load per edge
                               // (nullptr => single shard, row = u)
  int64_t pitch;               // elements per stored row (padded to 16 B)
  int dim;                     // logical columns to aggregate
  int col0;                    // first column inside the stored row
  DType dtype;
  int64_t zrow;                // single-shard view (loc == nullptr): index of an all-zero row
                               // in base[0] (padding edges read it), -1 if there is none
};

// Edge source for aggregation: either an ELL (cnt + nbr global ids, fixed stride
// k; used for layer 1 straight from the sampler) or a CSR over local indices.
struct AggArgs {
  // ELL form (layer 1)
  const int32_t* cnt;
  const int32_t* nbr;
  int k;
  // CSR form (upper layers)
  const int32_t* indptr;
  const int32_t* indices;
  const float* x;              // [n_src x x_pitch] fp32 (CSR form) ...
  int64_t x_pitch;
  const uint16_t* xb;          // ... or bf16 rows (bf16 mode's hidden activations, reading R11), pitch x_pitch
  // optional per-edge filter (SNP partial sums): only sources u with part[u] == keep_part
  const int32_t* filt_part;
  int keep_part;
  const int32_t* deg_override; // SNP: divide by the full sampled degree of the requester
  // rows
  const int32_t* n_dst;
  int64_t max_dst;
  int dim;
  // outputs (any may be null)
  float* z_f32;
  int64_t z_f32_pitch;
  uint16_t* z_bf16;
  int64_t z_bf16_pitch;
  int z_ones;                  // write 1.0 into bf16 column `dim` (bias-gradient column of the wgrad GEMM)
  int bpsm;                    // > 0: grid capped at this many blocks per SM (a background launch that
                               //   leaves registers for the step's chain beside it)
};
cudaError_t launch_agg_fstore(const AggArgs& a, const FeatView& fv, cudaStream_t st);
cudaError_t launch_agg_csr(const AggArgs& a, cudaStream_t st);

// dX[src_e] += dZ[v] / deg(v)  (O5 backward), fp32 atomics.
cudaError_t launch_agg_bwd(const int32_t* indptr, const int32_t* indices, const int32_t* n_dst, int64_t max_dst,
                           const float* dz, int64_t dz_pitch, int dim, float* dx, int64_t dx_pitch,
                           cudaStream_t st);

// Gather rows of the feature store into a dense buffer (apt_gather).
cudaError_t launch_gather(const FeatView& fv, const int32_t* ids, const int32_t* n_dev, int64_t max_n, void* out,
                          int64_t out_pitch, cudaStream_t st);

// Fill a shard with the synthetic O4 features of the listed global ids.
cudaError_t launch_fill_features(void* shard, DType dt, int64_t pitch, int col0, int ncols, const int32_t* ids,
                                 int64_t n, uint64_t seed, cudaStream_t st);

// ---------------------------------------------------------------- bwd.cu
// Transpose of a sampled block (counting sort): csc_ptr [n_src+1], csc_dst [E].
struct CscArgs {
  const int32_t* indptr; const int32_t* indices;
  const int32_t* n_dst; int64_t max_dst;
  const int32_t* n_edges; int64_t max_edges;
  const int32_t* n_src; int64_t max_src;
  int32_t* cnt;        // [max_src], zero on entry and exit
  int32_t* csc_ptr;    // [max_src + 1]
  int32_t* csc_total;  // [1]
  int2* csc_dst;       // [max_edges] (v, deg(v)) per in-edge
  int32_t* ws;         // scan workspace, >= 2*ceil(max_src/kScanWsTile) + 8
  int64_t grid_cap;    // max blocks of the grid-stride kernels (0: default)
  int k;               // > 0: rows have at most k edges (sampler fanout): fill by (row, slot) in parallel
  int counted;         // cnt already holds the in-degrees and the scan workspace is reset (launch_compact)
};
cudaError_t launch_csc_build(const CscArgs& a, cudaStream_t st);

// G[u] = mask(H[u] > 0) * sum_{(v,u)} dZ[v] / deg(v) over rows u < *n_src; fp32 G and/or
// bf16 Gb (whose 64-row-block tail is zeroed).
struct PullArgs {
  const int32_t* csc_ptr; const int2* csc_dst; const int32_t* indptr;
  const float* dz; int64_t dz_pitch;
  const float* h; int64_t h_pitch;        // null: no mask
  const uint16_t* mask; int64_t mask_pitch;   // if set: the ReLU mask as bits (replaces reading h)
  float* g; int64_t g_pitch;               // may be null
  uint16_t* gb; int64_t gb_pitch;          // may be null
  const int32_t* n_src; int64_t max_src;
  int dim;
  int dz_scaled;                           // dz rows already divided by deg (tcgen05 epilogue)
  const uint16_t* hb; int64_t hb_pitch;    // if set: the ReLU mask from bf16 H (bf16 mode, reading R11)
  const uint16_t* dzb; int64_t dzb_pitch;  // if set: dZ / deg as bf16 rows instead of dz (reading R13)
};
cudaError_t launch_pull_bwd(const PullArgs& a, cudaStream_t st);

// ---------------------------------------------------------------- gemm_simt.cu
// C[m][n] (+)= sum_k A(m,k) B(k,n) (+ bias[n]) (relu), fp32 accumulate.
// A(m,k) = A[m*sam + k*sak]; B(k,n) = B[k*sbk + n*sbn]; M may live on device.
struct SimtGemmArgs {
  const void* A; DType a_t; int64_t sam, sak;
  const void* B; DType b_t; int64_t sbk, sbn;
  float* C; int64_t ldc;
  const float* bias;
  const int32_t* M_dev;        // if set, M = *M_dev (<= M)
  int64_t M; int N; int64_t K;
  int relu;
  int accumulate;              // atomically add into C (split-K)
  int64_t k_chunk;             // split-K chunk (0 => whole K)
  const int32_t* K_dev;        // if set, K = *K_dev (<= K)
  // optional row routing: row m goes to out_base[out_rank[m]] + out_row[m] * ldc
  float* const* out_base; const int32_t* out_rank; const int32_t* out_row;
  // optional bf16 output instead of C (tensor-core path only; the hidden activations, R11)
  uint16_t* Cb; int64_t ldcb;
};
cudaError_t launch_simt_gemm(const SimtGemmArgs& a, cudaStream_t st);
// gemm_tc_gen.cu: the same contract on tcgen05 (fp32: 3xTF32 on kind::tf32; bf16:
// kind::f16), any M, N, K; ones_col >= 0 routes output column ones_col to ones_out[m]
// (the bias gradient from an all-ones column of B).  tc_gen_supported: TMA-addressable.
int tc_gen_supported(const SimtGemmArgs& a);
cudaError_t launch_tc_gen_gemm(const SimtGemmArgs& a, int ones_col, float* ones_out, cudaStream_t st);

// ---------------------------------------------------------------- gemm_tc.cu
// tcgen05 projection: Y[m][n] = sum_k Z[m][k] W[n][k] + bias[n] (relu), bf16 in,
// fp32 accumulate in TMEM, fp32 out.  Z, W are K-major bf16 with 16-B pitches.
struct TcGemmArgs {
  const uint16_t* Z; int64_t z_pitch;  // A: [M_max x K] bf16 (K-major)
  const uint16_t* W; int64_t w_pitch;  // B: [N x K] bf16 (K-major), or [K x N] if w_mn
  int64_t M_max; const int32_t* M_dev; int N; int K;
  const float* bias; int relu;
  float* Y; int64_t y_pitch;
  // optional row routing (peer-store epilogue): row m goes to
  // out_base[out_rank[m]] + out_row[m] * y_pitch
  float* const* out_base; const int32_t* out_rank; const int32_t* out_row;
  int w_mn;                            // B stored N-contiguous (dZ = G W uses W [d_out x d_in] as is)
  int accumulate;                      // add into Y with vector reductions (partial sums of SNP / NFP)
  uint16_t* mask; int64_t mask_pitch;  // optional: bit c%16 of mask[m][c/16] = (Y[m][c] > 0) (ReLU mask for the backward)
  // optional: row m is divided (RN) by its block degree indptr[m+1] - indptr[m] (the
  // mean's backward pre-scales dZ / deg once per row instead of once per in-edge)
  const int32_t* row_div_indptr;
  // optional bf16 output instead of Y (hidden activations in bf16 mode, reading R11):
  // row m -> Yb + m * yb_pitch (not with routing / accumulation)
  uint16_t* Yb; int64_t yb_pitch;
  int b_early;                         // W is not written by the preceding kernel (the step's projections)
};
int tc_gemm_supported(int N, int K);
cudaError_t launch_tc_gemm(const TcGemmArgs& a, cudaStream_t st);

// tcgen05 weight gradient: dW[o][i] += sum_r G[r][o] Z[r][i]; db[o] += sum_r G[r][o]
// (db via Z's all-ones column d_in, required when db != null).  G, Z bf16 row-major;
// rows beyond *rows_dev up to the next multiple of 64 must be zero in G.
struct TcWgradArgs {
  const uint16_t* G; int64_t g_pitch;  // [rows_max x d_out]
  const uint16_t* Z; int64_t z_pitch;  // [rows_max x (d_in + 1)]
  const int32_t* rows_dev; int64_t rows_max;
  int d_out, d_in;
  float* dW; float* db;
  int64_t ldw;                         // row stride of dW (0 => d_in)
};
int tc_wgrad_supported(int d_out, int d_in);
cudaError_t launch_tc_wgrad(const TcWgradArgs& a, cudaStream_t st);

// Gb = bf16(G * (H > 0)) over rows < n (relu != 0) or bf16(G); rows in
// [n, round_up(n, 64)) of Gb are zeroed (tail of the tcgen05 row blocks).
cudaError_t launch_grad_finish(const float* G, int64_t g_pitch, const float* H, int64_t h_pitch, int dim, int relu,
                               uint16_t* Gb, int64_t gb_pitch, const int32_t* n_dev, int64_t max_n, cudaStream_t st,
                               const uint16_t* Hb = nullptr, int64_t hb_pitch = 0);   // Hb: mask from bf16 H

// ---------------------------------------------------------------- misc.cu
cudaError_t launch_ce_loss(const float* logits, int64_t pitch, int n_classes, const int32_t* seeds,
                           const int32_t* n_seeds, int64_t max_seeds, const int32_t* labels,
                           const int32_t* n_global, float* loss, float* g, int64_t g_pitch, uint16_t* gb,
                           int64_t gb_pitch, float* zero, int64_t zero_n, int32_t* ws, cudaStream_t st);
// outfused.cu: the output layer's mean + projection + softmax CE in one kernel (bf16 mode)
struct OutFusedArgs {
  const int32_t* indptr; const int32_t* indices;       // the hop-0 block (CSR over H^{K-1} rows)
  const uint16_t* hb; int64_t hb_pitch;                 // H^{K-1} in bf16 (reading R11)
  const int32_t* n_dst; int64_t max_dst;
  int d_in, C;
  uint16_t* zb; int64_t zb_pitch;                       // Z^K (bf16, + the all-ones column d_in)
  const uint16_t* wb; int64_t wb_pitch;                 // W^K bf16 [C][wb_pitch]
  const float* bias;
  float* logits; int64_t l_pitch;                       // H^K (fp32)
  const int32_t* seeds; const int32_t* labels; const int32_t* n_global;
  float* loss; float* g; int64_t g_pitch; uint16_t* gb; int64_t gb_pitch;
  float* zero; int64_t zero_n; float* part; int32_t* ticket;
  uint16_t* dzb; int64_t dzb_pitch;                     // optional: dZ^K = (G W) / deg in bf16 (R13)
};
int out_fused_supported(int d_in, int C, int64_t max_dst);
cudaError_t launch_out_fused(const OutFusedArgs& a, cudaStream_t st);

// ce_loss workspace: [ticket, partial sums of up to kCeMaxBlocks blocks], zero-initialised once
constexpr int kCeMaxBlocks = 1024;
cudaError_t launch_relu_bwd(float* g, const float* h, int64_t pitch, int dim, const int32_t* n_dev, int64_t max_n,
                            cudaStream_t st);
cudaError_t launch_colsum(const float* g, int64_t pitch, int dim, const int32_t* n_dev, int64_t max_n, float* out,
                          cudaStream_t st);
cudaError_t launch_sgd(float* W, const float* dW, int64_t n, float lr, uint16_t* W_bf16, int rows, int cols,
                       int64_t bf16_pitch, cudaStream_t st);
struct SgdSeg { float* W; const float* dW; int64_t n; uint16_t* Wb; int cols; int64_t bpitch; };
struct SgdBatch { SgdSeg seg[16]; int n; };
cudaError_t launch_sgd_multi(const SgdBatch& b, float lr, cudaStream_t st);
cudaError_t launch_to_bf16(const float* src, int64_t src_pitch, uint16_t* dst, int64_t dst_pitch, int cols,
                           const int32_t* n_dev, int64_t max_n, cudaStream_t st);
cudaError_t launch_bf16_pad_ones(const uint16_t* src, int64_t src_pitch, uint16_t* dst, int64_t dst_pitch, int cols,
                                 const int32_t* n_dev, int64_t max_n, cudaStream_t st);
cudaError_t launch_transpose(const float* src, int rows, int cols, float* dst, cudaStream_t st);

}  // namespace apt
