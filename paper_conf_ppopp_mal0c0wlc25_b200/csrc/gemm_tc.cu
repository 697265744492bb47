// gemm_tc.cu -- S8: the dense projection Y = Z W^T + b (Fig. 5 "dense
// tensor multiplication between H^0 and W") on the 5th-generation tensor cores.
//
// sm_100a design:
//  * persistent CTAs (grid <= 148), one 128-row M tile per iteration;
//  * warp 0: TMA producer.  W (N x K, bf16, <= 256 x 256) is loaded once per CTA
//    and stays resident in shared memory; Z tiles (128 x 64 bf16, 128B swizzle)
//    stream through a 4-stage mbarrier ring;
//  * warp 1: TMEM allocator + single-thread tcgen05.mma issuer
//    (kind::f16, M=128, N=BN, K=16 per instruction), accumulators double
//    buffered in TMEM (2 x BN fp32 columns) so the epilogue of tile i overlaps
//    the MMAs of tile i+1;
//  * warps 2..5: epilogue.  tcgen05.ld 32x32b.x16 -> +bias -> ReLU -> fp32
//    stores; a row can be routed to another rank's buffer (peer-store epilogue
//    used by the DNP / SNP / NFP reshuffle).
// The projection is HBM-bound (AI <= 114 FLOP/B < ridge ~250), so the design
// goal is streaming Z and Y at full bandwidth, not MMA throughput.
#include "common.cuh"
#include "kernels.h"
#include <cuda.h>
#include <cudaTypedefs.h>
#include <algorithm>
#include <mutex>

namespace apt {

namespace tc {

constexpr int BM = 128;
constexpr int BK = 64;              // 64 bf16 = 128 B = one swizzle row
constexpr int STAGES = 4;
constexpr int A_STAGE_BYTES = BM * BK * 2;   // 16 KB
constexpr int THREADS = 192;        // 6 warps

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(b)), "r"(parity)
        : "memory");
  } while (!done);
}

__device__ __forceinline__ void tma_load_2d(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int x, int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// K-major operand, 128-byte swizzle: 8-row x 128-B atoms, SBO = 1024 B between
// atoms along M/N, LBO unused (1), descriptor version 1 (sm_100), layout 2.
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  return uint64_t((saddr & 0x3FFFFu) >> 4) | (uint64_t(1) << 16) | (uint64_t(1024 >> 4) << 32) |
         (uint64_t(1) << 46) | (uint64_t(2) << 61);
}

__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(accum)
      : "memory");
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

struct Params {
  int64_t M_max;
  const int32_t* M_dev;
  int N, BN, nkb, tmem_cols;
  const float* bias;
  int relu;
  float* Y;
  int64_t y_pitch;
  float* const* out_base;
  const int32_t* out_rank;
  const int32_t* out_row;
};

__global__ void __launch_bounds__(THREADS, 1)
    proj_kernel(const __grid_constant__ CUtensorMap mapZ, const __grid_constant__ CUtensorMap mapW, Params p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-B align the dynamic smem base (SWIZZLE_128B atoms)
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* smem_a = smem;                                        // STAGES x 16 KB
  uint8_t* smem_w = smem + STAGES * A_STAGE_BYTES;               // nkb x BN x 128 B
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_w + size_t(p.nkb) * p.BN * 128);
  uint64_t* full = bars;                  // [STAGES]
  uint64_t* empty = bars + STAGES;        // [STAGES]
  uint64_t* wfull = bars + 2 * STAGES;    // [1]
  uint64_t* tfull = wfull + 1;            // [2]
  uint64_t* tempty = tfull + 2;           // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int64_t M = std::min<int64_t>(p.M_max, int64_t(*p.M_dev));
  const int64_t ntiles = ceil_div(M, BM);

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    mbar_init(wfull, 1);
    for (int a = 0; a < 2; ++a) { mbar_init(tfull + a, 1); mbar_init(tempty + a, 128); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapZ)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapW)) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(uint32_t(p.tmem_cols)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ---- TMA producer
      mbar_expect_tx(wfull, uint32_t(p.nkb) * p.BN * 128);
      for (int kb = 0; kb < p.nkb; ++kb) tma_load_2d(smem_w + size_t(kb) * p.BN * 128, &mapW, wfull, kb * BK, 0);
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        for (int kb = 0; kb < p.nkb; ++kb) {
          mbar_wait(empty + s, ph ^ 1);
          mbar_expect_tx(full + s, A_STAGE_BYTES);
          tma_load_2d(smem_a + s * A_STAGE_BYTES, &mapZ, full + s, kb * BK, int(t * BM));
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ---- MMA issuer (one thread)
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(p.BN >> 3) << 17) | (uint32_t(BM >> 4) << 24);
    mbar_wait(wfull, 0);
    fence_after();
    int s = 0;
    uint32_t ph = 0;
    int acc = 0;
    uint32_t aph = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      mbar_wait(tempty + acc, aph ^ 1);
      fence_after();
      const uint32_t d = tmem_base + uint32_t(acc * p.BN);
      for (int kb = 0; kb < p.nkb; ++kb) {
        mbar_wait(full + s, ph);
        fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(smem_a + s * A_STAGE_BYTES);
          const uint32_t b0 = smem_u32(smem_w + size_t(kb) * p.BN * 128);
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk)
            mma_bf16(d, sw128_desc(a0 + kk * 32), sw128_desc(b0 + kk * 32), idesc, (kb | kk) != 0);
          mma_commit(empty + s);            // frees the smem stage when these MMAs finish
        }
        __syncwarp();
        if (++s == STAGES) { s = 0; ph ^= 1; }
      }
      if (lane == 0) mma_commit(tfull + acc);   // accumulator ready for the epilogue
      __syncwarp();
      acc ^= 1;
      if (acc == 0) aph ^= 1;
    }
  } else {
    // ---- epilogue warps 2..5: TMEM lane quarter = warp % 4
    const int q = warp & 3;
    int acc = 0;
    uint32_t aph = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      mbar_wait(tfull + acc, aph);
      fence_after();
      const int64_t m = t * BM + q * 32 + lane;
      const bool valid = m < M;
      float* out = nullptr;
      if (valid) {
        if (p.out_rank) out = p.out_base[p.out_rank[m]] + int64_t(p.out_row[m]) * p.y_pitch;
        else out = p.Y + m * p.y_pitch;
      }
      for (int c = 0; c < p.BN; c += 16) {
        uint32_t r[16];
        tmem_ld16(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * p.BN + c), r);
        if (!valid) continue;
        float v[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          float x = __uint_as_float(r[j]);
          if (p.bias && c + j < p.N) x += p.bias[c + j];
          if (p.relu) x = fmaxf(x, 0.f);
          v[j] = x;
        }
        if (c + 16 <= p.N) {
#pragma unroll
          for (int j = 0; j < 16; j += 4) *reinterpret_cast<float4*>(out + c + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
        } else {
          for (int j = 0; j < 16 && c + j < p.N; ++j) out[c + j] = v[j];
        }
      }
      fence_before();
      mbar_arrive(tempty + acc);
      acc ^= 1;
      if (acc == 0) aph ^= 1;
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(uint32_t(p.tmem_cols)));
  }
}

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
  });
  return fn;
}

static bool make_map(CUtensorMap* m, const void* base, int64_t cols, int64_t rows, int64_t pitch_elems, int box_cols,
                     int box_rows) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {cuuint64_t(cols), cuuint64_t(rows)};
  cuuint64_t strides[1] = {cuuint64_t(pitch_elems * 2)};
  cuuint32_t box[2] = {cuuint32_t(box_cols), cuuint32_t(box_rows)};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace tc

int tc_gemm_supported(int N, int K) { return N >= 1 && N <= 256 && K >= 1 && K <= 256; }

static int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

cudaError_t launch_tc_gemm(const TcGemmArgs& a, cudaStream_t st) {
  using namespace tc;
  if (!tc_gemm_supported(a.N, a.K)) return cudaErrorInvalidValue;
  if ((a.z_pitch * 2) % 16 || (a.w_pitch * 2) % 16 || (a.y_pitch * 4) % 16) return cudaErrorInvalidValue;
  const int BN = int(round_up(a.N, 16));
  const int nkb = int(ceil_div(a.K, BK));
  int cols = 32;
  while (cols < 2 * BN) cols <<= 1;
  CUtensorMap mz, mw;
  if (!make_map(&mz, a.Z, a.K, std::max<int64_t>(a.M_max, 1), a.z_pitch, BK, BM)) return cudaErrorInvalidValue;
  if (!make_map(&mw, a.W, a.K, a.N, a.w_pitch, BK, BN)) return cudaErrorInvalidValue;
  Params p{a.M_max, a.M_dev, a.N, BN, nkb, cols, a.bias, a.relu, a.Y, a.y_pitch, a.out_base, a.out_rank, a.out_row};
  const size_t smem = 1024 + size_t(STAGES) * A_STAGE_BYTES + size_t(nkb) * BN * 128 + 16 * 8 + 16;
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(proj_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set = true;
  }
  const int64_t tiles = std::max<int64_t>(1, ceil_div(a.M_max, BM));
  const int grid = int(std::min<int64_t>(tiles, sm_count()));
  proj_kernel<<<grid, THREADS, smem, st>>>(mz, mw, p);
  return cudaGetLastError();
}

}  // namespace apt
