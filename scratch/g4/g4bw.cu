// TMA gather4 throughput: each CTA (one per SM) streams random rows into a ring of
// NB chunk buffers (48 gather4 each), NW producer warps, consumer = mbarrier wait only.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait(uint64_t* b, uint32_t ph) {
  uint32_t done = 0;
  while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(su32(b)), "r"(ph) : "memory");
}
template <int NB, int NW>
__global__ void k(const __grid_constant__ CUtensorMap m, const int* ids, int chunks_per_cta, int rb) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t full[NB];
  const int G = 48;                  // gather4 per chunk
  const uint32_t slot = 896, cb = G * slot;
  if (threadIdx.x == 0) { for (int i = 0; i < NB; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(full + i))); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int c = 0; c < chunks_per_cta; ++c) {
    const int b = c % NB; const uint32_t ph = (c / NB) & 1;
    if (c >= NB) wait(full + b, ph ^ 1);   // previous use complete (consumer = us)
    if (warp == 0 && lane == 0) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(full + b)), "r"(G * 4 * rb) : "memory");
    __syncthreads();
    const int* cid = ids + ((size_t)(blockIdx.x * chunks_per_cta + c) * G * 4);
    for (int g = warp * 32 + lane; g < G; g += NW * 32) {
      int4 r = *reinterpret_cast<const int4*>(cid + g * 4);
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                   :: "r"(su32(sm + b * cb + g * slot)), "l"((uint64_t)&m), "r"(0), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w), "r"(su32(full + b)) : "memory");
    }
  }
  for (int c = chunks_per_cta - NB; c < chunks_per_cta; ++c) if (c >= 0) wait(full + (c % NB), (c / NB) & 1);
}
int main() {
  const int n = 2400000, cols = 104, rb = cols * 2;
  uint16_t* d; cudaMalloc(&d, (size_t)n * rb); cudaMemset(d, 1, (size_t)n * rb);
  const int ctas = 148, chunks = 21;     // ~ products layer 1: 148 x 21 x 192 rows ~ 600k rows
  const size_t nid = (size_t)ctas * chunks * 48 * 4;
  std::vector<int> h(nid); std::mt19937 rng(1); for (auto& x : h) x = rng() % n;
  int* di; cudaMalloc(&di, nid * 4); cudaMemcpy(di, h.data(), nid * 4, cudaMemcpyHostToDevice);
  void* f; cudaDriverEntryPointQueryResult q; cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  CUtensorMap m; cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)n}; cuuint64_t st[1] = {(cuuint64_t)rb};
  cuuint32_t box[2] = {(cuuint32_t)cols, 1}, es[2] = {1, 1};
  ((PFN_cuTensorMapEncodeTiled_v12000)f)(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  char* fl; cudaMalloc(&fl, 256 << 20);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
#define RUN(NB, NW) { auto kk = k<NB, NW>; size_t sm = NB * 48 * 896; cudaFuncSetAttribute(kk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm); \
    float best = 1e9; for (int it = 0; it < 5; ++it) { cudaMemset(fl, it, 256 << 20); cudaEventRecord(e0); kk<<<ctas, NW * 32, sm>>>(m, di, chunks, rb); cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); if (it) best = ms < best ? ms : best; } \
    printf("NB=%d NW=%d: %.1f us, %.0f GB/s (%s)\n", NB, NW, best * 1e3, nid * (double)rb / (best * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError())); }
  RUN(2, 1) RUN(4, 1) RUN(2, 4) RUN(4, 4)
}
