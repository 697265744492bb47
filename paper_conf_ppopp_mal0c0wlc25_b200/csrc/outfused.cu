// outfused.cu -- the output layer's forward tail as ONE kernel (bf16 mode): the last
// mean (Eq. 1: z_v = mean of the sampled h^{K-1}_u), the output projection
// (logits = z W^T + b, no activation) and the softmax cross-entropy with its gradient
// G = (softmax - onehot) / B (S10).  Replaces agg_kernel -> rowtile_kernel ->
// ce_loss_kernel, three dependent launches on 1 k rows whose each cost was its launch,
// drain and first-load latency (~6 / 6 / 10 us in the step for ~5 MB of L2 traffic).
//
// A CTA owns 16 destination rows (one per warp; APT_OUT_ROWS=32: two) end to end, so no
// phase waits on another CTA:
//   0. (before griddepcontrol.wait) W^K (bf16, <= 64 x 256) into shared memory -- the
//      step's weights change only in the SGD at its end;
//   1. the mean: a warp per row, lane j owns the row's 16-byte vector j, in-edges summed
//      in CSR order in fp32 (8 source rows in flight) -- the same order and the same
//      mixed-precision adds as agg_kernel, the same reciprocal division (O5) and bf16
//      rounding (R5), so Z is bit-identical to the unfused path; Z goes to shared memory
//      and to global (with the all-ones bias-gradient column) for the weight gradient;
//   2. logits = Z W^T + b on mma.sync m16n8k16 (bf16 in, fp32 accumulate; 1 k x 256 x 47
//      is ~25 MFLOP: latency, not tensor throughput, bounds it), written as fp32 H^K;
//   3. per row (a warp): max, sum exp, loss term, G and its bf16 copy -- ce_loss_kernel's
//      arithmetic; the gradient buffer zeroing, the 64-row-block tail of Gb and the
//      deterministic last-block loss sum are kept from it.
#include "common.cuh"
#include "kernels.h"
#include <cstdlib>

namespace apt {

namespace {
constexpr int kWarps = 16;
constexpr int kKMax = 256;         // d_in (multiple of 8)
constexpr int kNMax = 64;          // classes
constexpr int kSP = kKMax + 8;     // shared row stride (bf16): 528 B, conflict-free fragment loads
constexpr int kGS = kNMax + 8;     // G row stride (bf16): 144 B
constexpr int kEB = 8;             // source rows in flight per warp in the mean (a fanout-10 row: 8 + 2)

__device__ __forceinline__ void mma_bf16_16816(float* c, const uint32_t* a, const uint32_t* b) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}
}  // namespace

template <int kRows>   // destination rows per CTA (16 or 32)
__global__ void __launch_bounds__(kWarps * 32, 1) out_fused_kernel(OutFusedArgs a) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint16_t* Zs = reinterpret_cast<uint16_t*>(smem);                       // [kRows][kSP]
  uint16_t* Ws = Zs + kRows * kSP;                                         // [Cpad][kSP]
  const int Cpad = (a.C + 15) & ~15;
  float* Ls = reinterpret_cast<float*>(Ws + Cpad * kSP);                   // [kRows][kNMax + 1]
  __shared__ __align__(16) uint16_t Gs[kRows * kGS];                       // bf16 G (dZ = G W)
  __shared__ float degs[kRows];
  __shared__ float wsum[kWarps];
  __shared__ bool last;
  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int V = a.d_in >> 3;                                               // 16-byte vectors per row
  // 0. W^K into shared memory (rows past C zero), before the dependency wait
  for (int t = threadIdx.x; t < Cpad * V; t += blockDim.x) {
    const int n = t / V, j = t - n * V;
    uint4 w = make_uint4(0, 0, 0, 0);
    if (n < a.C) w = __ldg(reinterpret_cast<const uint4*>(a.wb + int64_t(n) * a.wb_pitch + j * 8));
    *reinterpret_cast<uint4*>(Ws + n * kSP + j * 8) = w;
  }
  pdl_wait();
  pdl_launch();
  const int64_t n = *a.n_dst;
  const int64_t r0 = int64_t(blockIdx.x) * kRows;
  // labels of this CTA's rows first (two dependent loads each): they land during the mean
  int y[kRows / kWarps];
#pragma unroll
  for (int q = 0; q < kRows / kWarps; ++q) {
    const int64_t i = r0 + warp + q * kWarps;
    y[q] = i < n ? a.labels[a.seeds[i]] : 0;
  }
  // 1. the mean
  uint64_t hbase;   // the lane's column base in H^{K-1} (lanes past the row's vectors: vector 0)
  asm("mov.b64 %0, %1;" : "=l"(hbase) : "l"(reinterpret_cast<uint64_t>(a.hb) + uint64_t(lane < V ? lane : 0) * 16u));
  const uint32_t hrb = uint32_t(a.hb_pitch * 2);
#pragma unroll 1
  for (int q = 0; q < kRows / kWarps; ++q) {
    const int rl = warp + q * kWarps;
    const int64_t i = r0 + rl;
    float acc[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) acc[k] = 0.f;
    int cnt = 0;
    if (i < n) {
      const int e0 = a.indptr[i];
      cnt = a.indptr[i + 1] - e0;
      for (int c0 = 0; c0 < cnt; c0 += 32) {
        const int u = c0 + lane < cnt ? a.indices[e0 + c0 + lane] : 0;
        const int m = min(32, cnt - c0);
        for (int e = 0; e < m; e += kEB) {
          uint4 v[kEB];
#pragma unroll
          for (int qq = 0; qq < kEB; ++qq) {
            // always-valid rows (lanes past the count hold row 0): one IMAD.WIDE per edge,
            // padding zeroed by a select, the adds unconditional
            const uint32_t uu = __shfl_sync(0xffffffffu, uint32_t(u), (e + qq) & 31);
            const uint4 t = __ldg(reinterpret_cast<const uint4*>(hbase + uint64_t(uu) * hrb));
            v[qq] = e + qq < m ? t : make_uint4(0, 0, 0, 0);
          }
#pragma unroll
          for (int qq = 0; qq < kEB; ++qq) accumulate_bf16x8(acc, v[qq]);
        }
      }
    }
    uint4 zv = make_uint4(0, 0, 0, 0);
    if (lane == 0) degs[rl] = float(cnt);
    if (i < n) {
      const float fdeg = float(cnt);
      const float rdeg = fdeg > 0.f ? __frcp_rn(fdeg) : 0.f;
      float z[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) z[k] = fdeg > 0.f ? div_rn_rcp(acc[k], fdeg, rdeg) : 0.f;
      zv = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]), pack_bf16x2(z[4], z[5]), pack_bf16x2(z[6], z[7]));
      if (lane < V) *reinterpret_cast<uint4*>(a.zb + i * a.zb_pitch + lane * 8) = zv;
      if (lane == 0) a.zb[i * a.zb_pitch + a.d_in] = 0x3F80;   // 1.0: the bias-gradient column
    }
    if (lane < V) *reinterpret_cast<uint4*>(Zs + rl * kSP + lane * 8) = zv;
    else if (lane < kKMax / 8) *reinterpret_cast<uint4*>(Zs + rl * kSP + lane * 8) = make_uint4(0, 0, 0, 0);
  }
  __syncthreads();
  // 2. logits: 2 m-tiles x (Cpad / 8) n-tiles of m16n8, one tile per warp
  {
    const int g = lane >> 2, t4 = lane & 3;
    constexpr int MT = kRows / 16;
    for (int tile = warp; tile < MT * (Cpad / 8); tile += kWarps) {
      const int mt = tile % MT, nt = tile / MT;
      float c[4] = {0.f, 0.f, 0.f, 0.f};
      const uint16_t* A0 = Zs + (mt * 16 + g) * kSP + 2 * t4;
      const uint16_t* A1 = A0 + 8 * kSP;
      const uint16_t* B0 = Ws + (nt * 8 + g) * kSP + 2 * t4;
      for (int k0 = 0; k0 < a.d_in; k0 += 16) {
        uint32_t af[4], bfr[2];
        af[0] = *reinterpret_cast<const uint32_t*>(A0 + k0);
        af[1] = *reinterpret_cast<const uint32_t*>(A1 + k0);
        af[2] = *reinterpret_cast<const uint32_t*>(A0 + k0 + 8);
        af[3] = *reinterpret_cast<const uint32_t*>(A1 + k0 + 8);
        bfr[0] = *reinterpret_cast<const uint32_t*>(B0 + k0);
        bfr[1] = *reinterpret_cast<const uint32_t*>(B0 + k0 + 8);
        mma_bf16_16816(c, af, bfr);
      }
      const int col = nt * 8 + 2 * t4;
      const int row = mt * 16 + g;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int rr = row + 8 * h;
#pragma unroll
        for (int k = 0; k < 2; ++k)
          if (col + k < a.C) Ls[rr * (kNMax + 1) + col + k] = c[2 * h + k] + a.bias[col + k];
      }
    }
  }
  for (int t = threadIdx.x; t < kRows * kGS / 2; t += blockDim.x) reinterpret_cast<uint32_t*>(Gs)[t] = 0u;
  __syncthreads();
  // the step's gradient accumulators start at zero (ce_loss_kernel's duty)
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < a.zero_n; t += int64_t(gridDim.x) * blockDim.x)
    a.zero[t] = 0.f;
  // 3. loss and gradient, a warp per row (ce_loss_kernel's arithmetic)
  const float inv_n = 1.0f / float(max(1, *a.n_global));
  float wloss = 0.f;
#pragma unroll
  for (int q = 0; q < kRows / kWarps; ++q) {
    const int rl = warp + q * kWarps;
    const int64_t i = r0 + rl;
    if (i >= n) continue;
    const float* row = Ls + rl * (kNMax + 1);
    for (int c = lane; c < a.C; c += 32) a.logits[i * a.l_pitch + c] = row[c];
    float m = -INFINITY;
    for (int c = lane; c < a.C; c += 32) m = fmaxf(m, row[c]);
    m = warp_max(m);
    float s = 0.f;
    for (int c = lane; c < a.C; c += 32) s += expf(row[c] - m);
    s = warp_sum(s);
    const float lse = m + logf(s);
    wloss += (lse - row[y[q]]) * inv_n;
    for (int c = lane; c < a.C; c += 32) {
      const float p = expf(row[c] - lse);
      const float v = (p - (c == y[q] ? 1.f : 0.f)) * inv_n;
      a.g[i * a.g_pitch + c] = v;
      const uint16_t vb = bf16_bits(v);
      a.gb[i * a.gb_pitch + c] = vb;
      Gs[rl * kGS + c] = vb;
    }
  }
  // 4. (a.dzb) dZ = (G W) / deg in bf16 (reading R13) for the mean's backward: the same
  // bf16 G and W the tcgen05 dZ kernel multiplies, fp32 accumulation, the correctly
  // rounded division per row, RNE to bf16
  if (a.dzb) {
    __syncthreads();
    const int g = lane >> 2, t4 = lane & 3;
    for (int tile = warp; tile < (kRows / 16) * (a.d_in / 8); tile += kWarps) {
      const int mt = tile % (kRows / 16), nt = tile / (kRows / 16);
      const int ncol = nt * 8 + g;
      float c[4] = {0.f, 0.f, 0.f, 0.f};
      const uint16_t* A0 = Gs + (mt * 16 + g) * kGS + 2 * t4;
      const uint16_t* A1 = A0 + 8 * kGS;
      for (int k0 = 0; k0 < Cpad; k0 += 16) {
        uint32_t af[4], bfr[2];
        af[0] = *reinterpret_cast<const uint32_t*>(A0 + k0);
        af[1] = *reinterpret_cast<const uint32_t*>(A1 + k0);
        af[2] = *reinterpret_cast<const uint32_t*>(A0 + k0 + 8);
        af[3] = *reinterpret_cast<const uint32_t*>(A1 + k0 + 8);
        const uint16_t* Wc = Ws + (k0 + 2 * t4) * kSP + ncol;   // W[class][col]: classes run down rows
        bfr[0] = uint32_t(Wc[0]) | (uint32_t(Wc[kSP]) << 16);
        bfr[1] = uint32_t(Wc[8 * kSP]) | (uint32_t(Wc[9 * kSP]) << 16);
        mma_bf16_16816(c, af, bfr);
      }
      const int col = nt * 8 + 2 * t4;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int rl = mt * 16 + g + 8 * h;
        const int64_t i = r0 + rl;
        if (i >= n) continue;
        float v0 = c[2 * h], v1 = c[2 * h + 1];
        const float dg = degs[rl];
        if (dg > 0.f) {
          const float rd = __frcp_rn(dg);
          v0 = div_rn_rcp(v0, dg, rd);
          v1 = div_rn_rcp(v1, dg, rd);
        }
        *reinterpret_cast<uint32_t*>(a.dzb + i * a.dzb_pitch + col) = pack_bf16x2(v0, v1);
      }
    }
  }
  {   // zero the tail of the last 64-row block of Gb (tcgen05 weight gradient reads whole blocks)
    const int64_t tail_end = std::min<int64_t>(a.max_dst, round_up(n, 64));
    for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < (tail_end - n) * a.gb_pitch;
         t += int64_t(gridDim.x) * blockDim.x)
      a.gb[n * a.gb_pitch + t] = 0;
  }
  // loss = the blocks' partial sums, reduced by the last block in a fixed order
  if (lane == 0) wsum[warp] = wloss;
  __syncthreads();
  if (threadIdx.x == 0) {
    float b = 0.f;
    for (int w = 0; w < kWarps; ++w) b += wsum[w];
    a.part[blockIdx.x] = b;
    __threadfence();
    last = atomicAdd(a.ticket, 1) == int(gridDim.x) - 1;
  }
  __syncthreads();
  if (last && threadIdx.x < 32) {
    __threadfence();
    float tot = 0.f;
    for (int b = lane; b < int(gridDim.x); b += 32) tot += __ldcg(a.part + b);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, o);
    if (lane == 0) {
      *a.loss = tot;
      *a.ticket = 0;
    }
  }
}

int out_fused_supported(int d_in, int C, int64_t max_dst) {
  static const int on = [] { const char* v = std::getenv("APT_OUT_FUSED"); return v ? atoi(v) : 1; }();
  return on && d_in % 16 == 0 && d_in >= 16 && d_in <= kKMax && C >= 1 && C <= kNMax &&
         ceil_div(max_dst, 16) <= kCeMaxBlocks;
}

cudaError_t launch_out_fused(const OutFusedArgs& a, cudaStream_t st) {
  if (!out_fused_supported(a.d_in, a.C, a.max_dst)) return cudaErrorInvalidValue;
  // APT_OUT_ROWS: rows per CTA (16: one row per warp, 2x the CTAs; 32: two rows per warp)
  static const int rows = [] { const char* v = std::getenv("APT_OUT_ROWS"); return v ? atoi(v) : 16; }();
  const int R = rows == 32 ? 32 : 16;
  const int Cpad = (a.C + 15) & ~15;
  const size_t smem = size_t(R + Cpad) * kSP * 2 + size_t(R) * (kNMax + 1) * 4;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(out_fused_kernel<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    cudaFuncSetAttribute(out_fused_kernel<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    attr = true;
  }
  const int64_t grid = std::max<int64_t>(1, ceil_div(a.max_dst, R));
  if (R == 32) launch_pdl(out_fused_kernel<32>, dim3(grid), dim3(kWarps * 32), smem, st, a);
  else launch_pdl(out_fused_kernel<16>, dim3(grid), dim3(kWarps * 32), smem, st, a);
  return cudaGetLastError();
}

}  // namespace apt
