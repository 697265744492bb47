// gemm_simt.cu -- the generic contraction entry (launch_simt_gemm) and its CUDA-core
// fallback.  Operands that TMA can address go to the tensor cores (gemm_tc_gen.cu:
// 3xTF32 for the fp32 parity mode, kind::f16 for bf16 past the row-tile kernel's
// limits); what remains (mixed operand types, strides that are not 16-byte multiples)
// runs here in exact fp32 FMA: the projection (S8) and the backward contractions
// (S10/S11: dW = g^T Z, dZ = g W).
//
// C[m][n] (+)= sum_k A(m,k) B(k,n) (+bias[n]) (relu) with arbitrary element
// strides, 64x64 tiles, 16-deep k slabs in shared memory, 4x4 outputs per
// thread, optional split-K with fp32 atomics into a zeroed C.
#include "common.cuh"
#include "kernels.h"
#include <algorithm>
#include <cstdlib>

namespace apt {

constexpr int BM = 64, BN = 64, BK = 16;

template <typename T>
__device__ __forceinline__ float ldf(const T* p, int64_t i);
template <>
__device__ __forceinline__ float ldf<float>(const float* p, int64_t i) { return p[i]; }
template <>
__device__ __forceinline__ float ldf<uint16_t>(const uint16_t* p, int64_t i) {
  return __uint_as_float(uint32_t(p[i]) << 16);
}

template <typename TA, typename TB>
__global__ void __launch_bounds__(256) simt_gemm_kernel(SimtGemmArgs a) {
  APT_PDL_PROLOGUE();
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int64_t M = a.M_dev ? std::min<int64_t>(a.M, *a.M_dev) : a.M;
  const int64_t K = a.K_dev ? std::min<int64_t>(a.K, *a.K_dev) : a.K;
  const int64_t m0 = int64_t(blockIdx.x) * BM;
  const int n0 = blockIdx.y * BN;
  if (m0 >= M) return;
  const int64_t kc = a.k_chunk > 0 ? a.k_chunk : K;
  const int64_t kb = int64_t(blockIdx.z) * kc;
  if (kb >= K && blockIdx.z > 0) return;
  const int64_t ke = std::min<int64_t>(K, kb + kc);
  const TA* A = reinterpret_cast<const TA*>(a.A);
  const TB* B = reinterpret_cast<const TB*>(a.B);
  const int tid = threadIdx.x;
  const int tm = (tid % 16) * 4, tn = (tid / 16) * 4;
  float acc[4][4] = {};
  for (int64_t k0 = kb; k0 < ke; k0 += BK) {
    // A slab [BK x BM]
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int mm, kk;
      if (a.sam == 1) { mm = tid % 64; kk = tid / 64 + 4 * j; }
      else { kk = tid % 16; mm = tid / 16 + 16 * j; }
      const int64_t gm = m0 + mm, gk = k0 + kk;
      As[kk][mm] = (gm < M && gk < ke) ? ldf<TA>(A, gm * a.sam + gk * a.sak) : 0.f;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int nn, kk;
      if (a.sbn == 1) { nn = tid % 64; kk = tid / 64 + 4 * j; }
      else { kk = tid % 16; nn = tid / 16 + 16 * j; }
      const int64_t gn = n0 + nn, gk = k0 + kk;
      Bs[kk][nn] = (gn < a.N && gk < ke) ? ldf<TB>(B, gk * a.sbk + gn * a.sbn) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { av[i] = As[kk][tm + i]; bv[i] = Bs[kk][tn + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int64_t gm = m0 + tm + i;
    if (gm >= M) continue;
    float* crow = a.out_rank ? a.out_base[a.out_rank[gm]] + int64_t(a.out_row[gm]) * a.ldc : a.C + gm * a.ldc;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gn = n0 + tn + j;
      if (gn >= a.N) continue;
      float v = acc[i][j];
      if (a.bias && blockIdx.z == 0) v += a.bias[gn];
      if (a.accumulate) {
        atomicAdd(crow + gn, v);
      } else {
        if (a.relu) v = fmaxf(v, 0.f);
        crow[gn] = v;
      }
    }
  }
}

cudaError_t launch_simt_gemm(const SimtGemmArgs& a, cudaStream_t st) {
  if (a.relu && a.accumulate) return cudaErrorInvalidValue;
  // tensor cores whenever the operands are TMA-addressable (gemm_tc_gen.cu: 3xTF32 for
  // fp32, kind::f16 for bf16); APT_SIMT_GEMM=1 keeps these CUDA cores (A/B)
  static const int simt_only = [] { const char* v = std::getenv("APT_SIMT_GEMM"); return v ? atoi(v) : 0; }();
  if (!simt_only && tc_gen_supported(a)) return launch_tc_gen_gemm(a, -1, nullptr, st);
  const int64_t kc = a.k_chunk > 0 ? a.k_chunk : a.K;
  dim3 grid(unsigned(std::max<int64_t>(1, ceil_div(a.M, BM))), unsigned(ceil_div(a.N, BN)),
            unsigned(std::max<int64_t>(1, ceil_div(a.K, kc))));
  if (a.a_t == kF32 && a.b_t == kF32) launch_pdl(simt_gemm_kernel<float, float>, dim3(grid), dim3(256), 0, st, a);
  else if (a.a_t == kF32 && a.b_t == kBF16) launch_pdl(simt_gemm_kernel<float, uint16_t>, dim3(grid), dim3(256), 0, st, a);
  else if (a.a_t == kBF16 && a.b_t == kF32) launch_pdl(simt_gemm_kernel<uint16_t, float>, dim3(grid), dim3(256), 0, st, a);
  else launch_pdl(simt_gemm_kernel<uint16_t, uint16_t>, dim3(grid), dim3(256), 0, st, a);
  return cudaGetLastError();
}

}  // namespace apt
