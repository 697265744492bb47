// common.cuh -- shared device helpers for the APT B200 hot path (sm_100a only).
//
// Nothing here is shared with oracle/ (the CPU oracle has its own Philox).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include <map>
#include <mutex>
#include <tuple>

#ifndef __CUDACC__
#error "compile with nvcc -gencode arch=compute_100a,code=sm_100a"
#endif

namespace apt {

constexpr int kWarp = 32;
constexpr int kMaxLayers = 4;
constexpr int kMaxRanks = 8;

// ---------------------------------------------------------------- Philox ----
// Philox4x32-10 (Salmon et al. SC'11), the counter-based generator that keys
// every random draw of the method (reading Z2: the paper fixes no RNG).
// Domain separation: key = (seed_lo, seed_hi ^ DOMAIN).
constexpr uint32_t kDomSample = 0x53414D50u;
constexpr uint32_t kDomFeat = 0x46454154u;
constexpr uint32_t kDomPerm = 0x5045524Du;

__host__ __device__ __forceinline__ uint4 philox(uint4 c, uint2 k) {
#pragma unroll
  for (int i = 0; i < 10; ++i) {
    if (i) { k.x += 0x9E3779B9u; k.y += 0xBB67AE85u; }
#ifdef __CUDA_ARCH__
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
#else
    const uint64_t p0 = 0xD2511F53ull * c.x, p1 = 0xCD9E8D57ull * c.z;
    const uint32_t hi0 = uint32_t(p0 >> 32), lo0 = uint32_t(p0);
    const uint32_t hi1 = uint32_t(p1 >> 32), lo1 = uint32_t(p1);
#endif
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
  }
  return c;
}

__host__ __device__ __forceinline__ uint2 philox_key(uint64_t seed, uint32_t dom) {
  return make_uint2(uint32_t(seed), uint32_t(seed >> 32) ^ dom);
}

__host__ __device__ __forceinline__ uint32_t word_of(uint4 w, int i) {
  return i == 0 ? w.x : i == 1 ? w.y : i == 2 ? w.z : w.w;
}

// Synthetic feature x[u][j] = (int8)(Philox_FEAT(seed;{u,0,j>>2,0}).word(j&3)) / 64
// (input recipe O4; exact in bf16 and fp32).
__host__ __device__ __forceinline__ float feature_value(uint2 key, int64_t u, int j) {
  uint4 w = philox(make_uint4(uint32_t(u), uint32_t(uint64_t(u) >> 32), uint32_t(j >> 2), 0u), key);
  int8_t b = int8_t(word_of(w, j & 3) & 0xFFu);
  return float(b) * (1.0f / 64.0f);
}

// ------------------------------------------------- programmatic launches ----
// Every kernel of the step is launched with programmatic stream serialization:
// the next kernel's CTAs are scheduled while the previous kernel drains, and each
// kernel waits (griddepcontrol.wait = all predecessor grids complete and their
// memory visible) before touching anything, then immediately allows its own
// dependents to launch.  In a CUDA graph these become programmatic edges, which
// hides most of the per-kernel launch latency of a ~40-kernel step.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch() { asm volatile("griddepcontrol.launch_dependents;" :::); }
#define APT_PDL_PROLOGUE() do { ::apt::pdl_wait(); ::apt::pdl_launch(); } while (0)

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

// ------------------------------------------------------- grid sizing ----
// SM count of the current device (148 on B200), queried once per process (one process
// drives one device; an emulated job uses one device too).
inline int num_sms() {
  static const int n = [] {
    int d = 0, v = 0;
    if (cudaGetDevice(&d) != cudaSuccess || cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d) != cudaSuccess ||
        v <= 0)
      v = 148;
    return v;
  }();
  return n;
}
// Resident blocks per SM the hardware grants this kernel (registers, shared memory,
// launch bounds), queried once per instantiation: a "one resident wave" grid is
// num_sms() * resident_blocks(kernel, threads).
template <typename K>
inline int resident_blocks(K kernel, int threads, size_t smem = 0) {
  static std::mutex mu;
  static std::map<std::tuple<const void*, int, size_t>, int> cache;
  const auto key = std::make_tuple(reinterpret_cast<const void*>(kernel), threads, smem);
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(key);
  if (it != cache.end()) return it->second;
  int b = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, threads, smem) != cudaSuccess || b <= 0) b = 1;
  cache.emplace(key, b);
  return b;
}
// Grid of ceil(n / per_block) blocks capped at `per_sm` blocks on every SM.
inline int64_t grid_cap(int64_t want, int64_t per_sm) {
  const int64_t cap = int64_t(num_sms()) * per_sm;
  return want < 1 ? 1 : (want < cap ? want : cap);
}

// ---------------------------------------------------------------- misc ----
__host__ __device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
__host__ __device__ __forceinline__ int64_t round_up(int64_t a, int64_t b) { return ceil_div(a, b) * b; }

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ float bf16_lo(uint32_t v) { return __uint_as_float(v << 16); }
__device__ __forceinline__ float bf16_bits_to_float(uint16_t b) { return __uint_as_float(uint32_t(b) << 16); }
// acc0 += lo(w), acc1 += hi(w) for a packed bf16 pair: the mixed-precision add
// (add.rn.f32.bf16 -> FHADD.BF16 with an .H0/.H1 operand select) is one instruction per
// element where the unpack (shift / mask) + FADD form took two; the bf16 value converts to
// fp32 exactly, so the sums are bit-identical to the unpacked form
__device__ __forceinline__ void acc_bf16x2(float& a0, float& a1, uint32_t w) {
  asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %2;\n\t"
      "add.rn.f32.bf16 %0, lo, %0;\n\tadd.rn.f32.bf16 %1, hi, %1;\n\t}"
      : "+f"(a0), "+f"(a1) : "r"(w));
}

__device__ __forceinline__ void accumulate_bf16x8(float* acc, uint4 raw) {
  acc_bf16x2(acc[0], acc[1], raw.x); acc_bf16x2(acc[2], acc[3], raw.y);
  acc_bf16x2(acc[4], acc[5], raw.z); acc_bf16x2(acc[6], acc[7], raw.w);
}
__device__ __forceinline__ uint16_t bf16_bits(float x) {
  __nv_bfloat16 h = __float2bfloat16_rn(x);
  return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float bf16_hi(uint32_t v) { return __uint_as_float(v & 0xFFFF0000u); }

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);   // RNE (O5 rounding point)
  return *reinterpret_cast<uint32_t*>(&h);
}

// IEEE round-to-nearest x / d (reading O5) for d >= 1.  A zero numerator takes the
// division's slow path (exponent 0), so it is answered directly: 0 / d = 0 (same
// sign), which keeps every sum that cancels to zero off the ~100-instruction path.
__device__ __forceinline__ float div_rn(float x, float d) { return x == 0.f ? x : __fdiv_rn(x, d); }

// Correctly rounded x / d from a correctly rounded reciprocal r = RN(1/d)
// (Markstein: with r within 1/2 ulp of 1/d and q0 within 1 ulp of x/d, the
// residual rem = x - q0*d is exact in one FMA and q0 + rem*r rounds to RN(x/d)).
// Valid for normal x, d (all means of the method: |x| < 2^24, d in [1, 2^16]);
// checked exhaustively against __fdiv_rn by apt_selftest_div.
__device__ __forceinline__ float div_rn_rcp(float x, float d, float r) {
  const float q0 = x * r;
  const float rem = fmaf(-q0, d, x);
  return fmaf(rem, r, q0);
}

// 16-byte loads bypassing L1 allocation for streaming rows.
__device__ __forceinline__ uint4 ld_nc_v4(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// Vector fp32 atomic add (sm_90+): 4 floats per red.
// One 32-byte store (a whole L2 sector) per thread: st.global.v8.b32 -> STG.E.256 (sm_100).
__device__ __forceinline__ void st_v8(void* p, uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t a4,
                                      uint32_t a5, uint32_t a6, uint32_t a7) {
  asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(a0), "r"(a1), "r"(a2), "r"(a3),
               "r"(a4), "r"(a5), "r"(a6), "r"(a7)
               : "memory");
}

__device__ __forceinline__ void red_add_v4(float* p, float a, float b, float c, float d) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d)
               : "memory");
}

// Device error word: kernels OR an APT_DEV_* bit on invalid input instead of trapping.
enum : uint32_t { kDevErrBadId = 1u, kDevErrOverflow = 2u, kDevErrTimeout = 4u };

}  // namespace apt

#define APT_CUDA_OK(expr)                                                     \
  do {                                                                        \
    cudaError_t _e = (expr);                                                  \
    if (_e != cudaSuccess) return ::apt::fail_cuda(_e, #expr, __FILE__, __LINE__); \
  } while (0)
