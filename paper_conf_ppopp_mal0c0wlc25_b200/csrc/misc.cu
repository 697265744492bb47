// misc.cu -- small elementwise kernels of the training step (S10/S11):
// cross-entropy loss + its gradient, ReLU backward, bias gradient, SGD update
// with the bf16 weight copy for the tensor-core projection, conversions.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>

namespace apt {

static int64_t grid_of(int64_t n, int t = 256) {
  return grid_cap(ceil_div(n, t), 32);
}

// loss = sum_s CE(logits_s, y_s) / n_global  (reading Z20);  g = (softmax - onehot) / n_global.
__global__ void ce_loss_kernel(const float* __restrict__ logits, int64_t pitch, int C,
                               const int32_t* __restrict__ seeds, const int32_t* __restrict__ n_seeds_p,
                               const int32_t* __restrict__ labels, const int32_t* __restrict__ n_global_p,
                               float* __restrict__ loss, float* __restrict__ g, int64_t g_pitch,
                               uint16_t* __restrict__ gb, int64_t gb_pitch, int64_t max_seeds,
                               float* __restrict__ zero, int64_t zero_n, float* __restrict__ part,
                               int32_t* __restrict__ ticket) {
  APT_PDL_PROLOGUE();
  const int lane = lane_id();
  const int64_t n = *n_seeds_p;
  const float inv_n = 1.0f / float(max(1, *n_global_p));
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  // the step's gradient accumulators start at zero (the backward's reductions add into
  // them); done here instead of a memset node, which would break the PDL chain
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < zero_n; t += int64_t(gridDim.x) * blockDim.x)
    zero[t] = 0.f;
  float wloss = 0.f;   // this warp's rows (fixed assignment: the loss sum is deterministic)
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n; i += nwarps) {
    const float* row = logits + i * pitch;
    // the label's two dependent loads (seed id, then its label) are issued before the
    // row's arithmetic so that their latency overlaps it
    const int y = labels[seeds[i]];
    float m = -INFINITY;
    for (int c = lane; c < C; c += 32) m = fmaxf(m, row[c]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f;
    for (int c = lane; c < C; c += 32) s += expf(row[c] - m);
    s = warp_sum(s);
    const float lse = m + logf(s);
    wloss += (lse - row[y]) * inv_n;
    for (int c = lane; c < C; c += 32) {
      const float p = expf(row[c] - lse);
      const float v = (p - (c == y ? 1.f : 0.f)) * inv_n;
      g[i * g_pitch + c] = v;
      if (gb) {
        __nv_bfloat16 h = __float2bfloat16_rn(v);
        gb[i * gb_pitch + c] = *reinterpret_cast<uint16_t*>(&h);
      }
    }
  }
  if (gb) {   // zero the tail of the last 64-row block (tcgen05 wgrad reads whole blocks)
    const int64_t tail_end = std::min<int64_t>(max_seeds, round_up(n, 64));
    for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < (tail_end - n) * gb_pitch;
         t += int64_t(gridDim.x) * blockDim.x)
      gb[n * gb_pitch + t] = 0;
  }
  // loss = the blocks' partial sums, reduced by the last block to finish in a fixed order
  // (lane l adds blocks l, l+32, ... then a fixed shuffle tree): no zeroed accumulator
  // before the kernel, run-to-run identical, and the partials are read 32 at a time
  // rather than one dependent L2 round trip after another
  __shared__ float wsum[8];
  __shared__ bool last;
  if (lane == 0) wsum[threadIdx.x >> 5] = wloss;
  __syncthreads();
  if (threadIdx.x == 0) {
    float b = 0.f;
    for (int w = 0; w < int(blockDim.x >> 5); ++w) b += wsum[w];
    part[blockIdx.x] = b;
    __threadfence();
    last = atomicAdd(ticket, 1) == int(gridDim.x) - 1;
  }
  __syncthreads();
  if (last && threadIdx.x < 32) {
    __threadfence();
    float tot = 0.f;
    for (int b = lane; b < int(gridDim.x); b += 32) tot += __ldcg(part + b);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, o);
    if (lane == 0) {
      *loss = tot;
      *ticket = 0;
    }
  }
}

cudaError_t launch_ce_loss(const float* logits, int64_t pitch, int n_classes, const int32_t* seeds,
                           const int32_t* n_seeds, int64_t max_seeds, const int32_t* labels,
                           const int32_t* n_global, float* loss, float* g, int64_t g_pitch, uint16_t* gb,
                           int64_t gb_pitch, float* zero, int64_t zero_n, int32_t* ws, cudaStream_t st) {
  const int64_t grid = std::min<int64_t>(kCeMaxBlocks, grid_of(max_seeds * 32));
  launch_pdl(ce_loss_kernel, dim3(grid), dim3(256), 0, st, logits, pitch, n_classes, seeds, n_seeds, labels,
             n_global, loss, g, g_pitch, gb, gb_pitch, max_seeds, zero, zero_n, reinterpret_cast<float*>(ws + 1), ws);
  return cudaGetLastError();
}

__global__ void relu_bwd_kernel(float* __restrict__ g, const float* __restrict__ h, int64_t pitch, int dim,
                                const int32_t* __restrict__ n_p) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int64_t total = n * dim;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / dim;
    const int64_t off = r * pitch + (t - r * dim);
    if (!(h[off] > 0.f)) g[off] = 0.f;
  }
}

cudaError_t launch_relu_bwd(float* g, const float* h, int64_t pitch, int dim, const int32_t* n_dev, int64_t max_n,
                            cudaStream_t st) {
  launch_pdl(relu_bwd_kernel, dim3(grid_of(max_n * dim)), dim3(256), 0, st, g, h, pitch, dim, n_dev);
  return cudaGetLastError();
}

// Gb = bf16(G * (H > 0)) (or bf16(G)); the 64-row-block tail of Gb is zeroed.
// One thread per 4 columns (16-B G / H loads, 8-B Gb stores).
__global__ void grad_finish_kernel(const float* __restrict__ G, int64_t gp, const float* __restrict__ H, int64_t hp,
                                   int dim, int relu, uint16_t* __restrict__ Gb, int64_t gbp,
                                   const int32_t* __restrict__ n_p, int64_t max_n,
                                   const uint16_t* __restrict__ Hb, int64_t hbp) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int64_t rows = std::min<int64_t>(max_n, round_up(n, 64));
  const int V = int(ceil_div(dim, 4));
  const int64_t total = rows * V;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / V;
    const int c = int(t - r * V) * 4;
    uint16_t* o = Gb + r * gbp + c;
    if (r >= n) {
      for (int q = 0; q < 4 && c + q < dim; ++q) o[q] = 0;
      continue;
    }
    float4 g = *reinterpret_cast<const float4*>(G + r * gp + c);
    if (relu && Hb) {   // bf16 H: positive <=> sign bit clear and not zero
      const uint16_t* hb = Hb + r * hbp + c;
      if (!(hb[0] != 0 && !(hb[0] & 0x8000u))) g.x = 0.f;
      if (!(c + 1 < dim && hb[1] != 0 && !(hb[1] & 0x8000u))) g.y = 0.f;
      if (!(c + 2 < dim && hb[2] != 0 && !(hb[2] & 0x8000u))) g.z = 0.f;
      if (!(c + 3 < dim && hb[3] != 0 && !(hb[3] & 0x8000u))) g.w = 0.f;
    } else if (relu) {
      const float4 h = *reinterpret_cast<const float4*>(H + r * hp + c);
      if (!(h.x > 0.f)) g.x = 0.f;
      if (!(h.y > 0.f)) g.y = 0.f;
      if (!(h.z > 0.f)) g.z = 0.f;
      if (!(h.w > 0.f)) g.w = 0.f;
    }
    if (c + 4 <= dim && (gbp & 3) == 0) {
      *reinterpret_cast<uint2*>(o) = make_uint2(pack_bf16x2(g.x, g.y), pack_bf16x2(g.z, g.w));
    } else {
      const float v[4] = {g.x, g.y, g.z, g.w};
      for (int q = 0; q < 4 && c + q < dim; ++q) {
        __nv_bfloat16 h = __float2bfloat16_rn(v[q]);
        o[q] = *reinterpret_cast<uint16_t*>(&h);
      }
    }
  }
}

cudaError_t launch_grad_finish(const float* G, int64_t g_pitch, const float* H, int64_t h_pitch, int dim, int relu,
                               uint16_t* Gb, int64_t gb_pitch, const int32_t* n_dev, int64_t max_n, cudaStream_t st,
                               const uint16_t* Hb, int64_t hb_pitch) {
  if ((g_pitch & 3) || (h_pitch & 3)) return cudaErrorInvalidValue;
  launch_pdl(grad_finish_kernel, dim3(grid_of(max_n * ceil_div(dim, 4))), dim3(256), 0, st, G, g_pitch, H, h_pitch, dim, relu, Gb,
                                                                          gb_pitch, n_dev, max_n, Hb, hb_pitch);
  return cudaGetLastError();
}

// dst[r][0:cols] = src[r][0:cols], dst[r][cols] = 1.0 (bf16), zero tail rows to the 64-row block.
__global__ void bf16_pad_ones_kernel(const uint16_t* __restrict__ src, int64_t sp, uint16_t* __restrict__ dst,
                                     int64_t dp, int cols, const int32_t* __restrict__ n_p, int64_t max_n) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int64_t rows = std::min<int64_t>(max_n, round_up(n, 64));
  const int64_t total = rows * dp;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / dp;
    const int c = int(t - r * dp);
    dst[t] = r >= n ? 0 : c < cols ? src[r * sp + c] : c == cols ? 0x3F80 : 0;
  }
}

cudaError_t launch_bf16_pad_ones(const uint16_t* src, int64_t src_pitch, uint16_t* dst, int64_t dst_pitch, int cols,
                                 const int32_t* n_dev, int64_t max_n, cudaStream_t st) {
  launch_pdl(bf16_pad_ones_kernel, dim3(grid_of(max_n * dst_pitch)), dim3(256), 0, st, src, src_pitch, dst, dst_pitch, cols, n_dev, max_n);
  return cudaGetLastError();
}

// out[c] += sum_r g[r][c]  (db = sum of g over the rows, O5)
__global__ void colsum_kernel(const float* __restrict__ g, int64_t pitch, int dim, const int32_t* __restrict__ n_p,
                              float* __restrict__ out) {
  APT_PDL_PROLOGUE();
  const int64_t n = *n_p;
  const int c = blockIdx.y * blockDim.x + threadIdx.x;
  if (c >= dim) return;
  const int64_t rows_per = ceil_div(n, gridDim.x);
  const int64_t r0 = int64_t(blockIdx.x) * rows_per, r1 = std::min<int64_t>(n, r0 + rows_per);
  float s = 0.f;
  for (int64_t r = r0; r < r1; ++r) s += g[r * pitch + c];
  if (r1 > r0) atomicAdd(out + c, s);
}

cudaError_t launch_colsum(const float* g, int64_t pitch, int dim, const int32_t* n_dev, int64_t max_n, float* out,
                          cudaStream_t st) {
  const int tx = 128;
  dim3 grid(unsigned(std::max<int64_t>(1, std::min<int64_t>(max_n / 256 + 1, 296))), unsigned(ceil_div(dim, tx)));
  launch_pdl(colsum_kernel, dim3(grid), dim3(tx), 0, st, g, pitch, dim, n_dev, out);
  return cudaGetLastError();
}

// W -= lr * dW; optionally refresh the bf16 copy [rows x cols] (pitch) used by tcgen05.
__global__ void sgd_kernel(float* __restrict__ W, const float* __restrict__ dW, int64_t n, float lr,
                           uint16_t* __restrict__ wb, int cols, int64_t bpitch) {
  APT_PDL_PROLOGUE();
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < n; t += int64_t(gridDim.x) * blockDim.x) {
    const float w = W[t] - lr * dW[t];
    W[t] = w;
    if (wb) {
      const int64_t r = t / cols;
      __nv_bfloat16 h = __float2bfloat16_rn(w);
      wb[r * bpitch + (t - r * cols)] = *reinterpret_cast<uint16_t*>(&h);
    }
  }
}

// All parameter tensors of a step in one launch: blockIdx.y = tensor.
__global__ void sgd_multi_kernel(SgdBatch b, float lr) {
  APT_PDL_PROLOGUE();
  const SgdSeg& g = b.seg[blockIdx.y];
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < g.n; t += int64_t(gridDim.x) * blockDim.x) {
    const float w = g.W[t] - lr * g.dW[t];
    g.W[t] = w;
    if (g.Wb) {
      const int64_t r = t / g.cols;
      __nv_bfloat16 h = __float2bfloat16_rn(w);
      g.Wb[r * g.bpitch + (t - r * g.cols)] = *reinterpret_cast<uint16_t*>(&h);
    }
  }
}

cudaError_t launch_sgd_multi(const SgdBatch& b, float lr, cudaStream_t st) {
  if (b.n <= 0) return cudaSuccess;
  int64_t mx = 1;
  for (int i = 0; i < b.n; ++i) mx = std::max<int64_t>(mx, b.seg[i].n);
  dim3 grid(unsigned(grid_cap(ceil_div(mx, 256), 4)), unsigned(b.n));
  launch_pdl(sgd_multi_kernel, dim3(grid), dim3(256), 0, st, b, lr);
  return cudaGetLastError();
}

cudaError_t launch_sgd(float* W, const float* dW, int64_t n, float lr, uint16_t* W_bf16, int rows, int cols,
                       int64_t bf16_pitch, cudaStream_t st) {
  (void)rows;
  launch_pdl(sgd_kernel, dim3(grid_of(n)), dim3(256), 0, st, W, dW, n, lr, W_bf16, cols, bf16_pitch);
  return cudaGetLastError();
}

__global__ void to_bf16_kernel(const float* __restrict__ src, int64_t sp, uint16_t* __restrict__ dst, int64_t dp,
                               int cols, const int32_t* __restrict__ n_p, int64_t n_static) {
  APT_PDL_PROLOGUE();
  const int64_t n = n_p ? int64_t(*n_p) : n_static;
  const int64_t total = n * cols;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < total; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / cols;
    const int c = int(t - r * cols);
    __nv_bfloat16 h = __float2bfloat16_rn(src[r * sp + c]);
    dst[r * dp + c] = *reinterpret_cast<uint16_t*>(&h);
  }
}

cudaError_t launch_to_bf16(const float* src, int64_t src_pitch, uint16_t* dst, int64_t dst_pitch, int cols,
                           const int32_t* n_dev, int64_t max_n, cudaStream_t st) {
  launch_pdl(to_bf16_kernel, dim3(grid_of(max_n * cols)), dim3(256), 0, st, src, src_pitch, dst, dst_pitch, cols, n_dev, max_n);
  return cudaGetLastError();
}

__global__ void transpose_kernel(const float* __restrict__ s, int rows, int cols, float* __restrict__ d) {
  const int64_t n = int64_t(rows) * cols;
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < n; t += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = t / cols;
    const int c = int(t - r * cols);
    d[int64_t(c) * rows + r] = s[t];
  }
}

cudaError_t launch_transpose(const float* src, int rows, int cols, float* dst, cudaStream_t st) {
  transpose_kernel<<<grid_of(int64_t(rows) * cols), 256, 0, st>>>(src, rows, cols, dst);
  return cudaGetLastError();
}

}  // namespace apt

namespace apt {
// Node ids are int64 at the ABI and int32 inside (n_nodes < 2^31).
__global__ void widen_ids_kernel(const int32_t* __restrict__ a, int64_t n, int64_t* __restrict__ b) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) b[i] = a[i];
}
__global__ void narrow_ids_kernel(const int64_t* __restrict__ a, int64_t n, int64_t n_nodes, int32_t* __restrict__ b,
                                  uint32_t* err) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t v = a[i];
    if (v < 0 || v >= n_nodes) {
      atomicOr(err, kDevErrBadId);
      b[i] = 0;
    } else {
      b[i] = int32_t(v);
    }
  }
}
cudaError_t launch_widen_ids(const int32_t* a, int64_t n, int64_t* b, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  widen_ids_kernel<<<unsigned(grid_cap(ceil_div(n, 256), 16)), 256, 0, st>>>(a, n, b);
  return cudaGetLastError();
}
cudaError_t launch_narrow_ids(const int64_t* a, int64_t n, int64_t n_nodes, int32_t* b, uint32_t* err, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  narrow_ids_kernel<<<unsigned(grid_cap(ceil_div(n, 256), 16)), 256, 0, st>>>(a, n, n_nodes, b, err);
  return cudaGetLastError();
}
}  // namespace apt
