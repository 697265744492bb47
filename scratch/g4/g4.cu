// micro-test: TMA tile::gather4 semantics on sm_100a
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k(const __grid_constant__ CUtensorMap m, int r0, int r1, int r2, int r3, int cols, uint16_t* out) {
  __shared__ __align__(1024) uint16_t buf[4 * 256];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar)), "r"(4 * cols * 2) : "memory");
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 :: "r"(su32(buf)), "l"((uint64_t)&m), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(&bar)) : "memory");
  }
  uint32_t done = 0;
  while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(su32(&bar)) : "memory");
  for (int i = threadIdx.x; i < 4 * cols; i += blockDim.x) out[i] = buf[i];
}

int main() {
  const int n = 1000, cols = 104;
  std::vector<uint16_t> h(n * cols);
  for (int r = 0; r < n; ++r) for (int c = 0; c < cols; ++c) h[r * cols + c] = uint16_t(r * 10 + (c % 10));
  uint16_t *d, *o;
  cudaMalloc(&d, h.size() * 2); cudaMalloc(&o, 4 * 256 * 2);
  cudaMemcpy(d, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
  void* f = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)f;
  CUtensorMap m;
  for (int boxr : {1, 4}) {
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)n};
    cuuint64_t str[1] = {(cuuint64_t)cols * 2};
    cuuint32_t box[2] = {(cuuint32_t)cols, (cuuint32_t)boxr};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("box rows %d encode %d\n", boxr, (int)r);
    if (r) continue;
    cudaMemset(o, 0, 4 * 256 * 2);
    k<<<1, 128>>>(m, 5, 100, 7, 999, cols, o);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel %s\n", cudaGetErrorString(e));
    std::vector<uint16_t> ho(4 * cols);
    cudaMemcpy(ho.data(), o, ho.size() * 2, cudaMemcpyDeviceToHost);
    for (int i = 0; i < 4; ++i) printf("row %d: %d %d ... %d\n", i, ho[i * cols], ho[i * cols + 1], ho[i * cols + cols - 1]);
    if (e) break;
  }
}
