// gemm_tc_gen.cu -- the general tcgen05 contraction of the step: every GEMM the
// row-tile / weight-gradient kernels of gemm_tc.cu do not cover, on tensor cores.
//
//   C[m][n] (+)= sum_k A(m, k) B(k, n)  (+ bias[n]) (ReLU)          (S8, S10, S11)
//
// with A, B each either K-major or M/N-major in memory (element strides 1 and a 16-byte
// multiple), M and K optionally device-counted, N tiled in <= 256-column slices and K
// streamed (no size limit on either), split-K with fp32 vector reductions, and the
// routed / accumulating epilogues of the strategies.  Two operand types:
//
//  * fp32 (the parity mode, reading P1 of DESIGN.md): 3xTF32 on kind::tf32.  Every
//    operand tile is split in shared memory into x_hi = RN_tf32(x) (in place) and
//    x_lo = x - x_hi (exact in fp32, a second buffer); the tile contributes
//    A_hi B_hi + A_lo B_hi + A_hi B_lo (three MMAs per K=8 slice), so each product is
//    carried to ~2^-21 of its magnitude (the dropped A_lo B_lo and the tensor core's
//    reading of x_lo at TF32 width are both ~2^-22), well inside fp32's T1 bar;
//  * bf16: kind::f16, one pass (operands already carry the bf16 rounding points).
//
// sm_100a structure (persistent CTAs over (m, n, k-split) tiles, 14 warps):
//   warp 0      TMA producer: A and B tiles of one 128-byte swizzle atom of K per stage
//               (32 fp32 / 64 bf16), SW128, mbarrier ring;
//   warp 1      TMEM allocator + single-thread MMA issuer (M = 128, N = BN), double-
//               buffered accumulators so a tile's epilogue overlaps the next tile's MMAs;
//   warps 2-5   (fp32) the hi / lo split of every stage, and the zeroing of rows past a
//               device-counted K (stale rows of a reused buffer);
//   warps 6-13  epilogue: tcgen05.ld 32x32b chunks of 16 columns -> bias / ReLU ->
//               fp32 rows (routed to the requester's buffer, or reduced with red.v4).
#include "common.cuh"
#include "kernels.h"
#include "tc_common.cuh"
#include <cuda.h>
#include <cudaTypedefs.h>
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

namespace apt {
namespace tcg {

using tc::fence_after;
using tc::fence_before;
using tc::mbar_arrive;
using tc::mbar_expect_tx;
using tc::mbar_init;
using tc::mbar_wait;
using tc::mma_commit;
using tc::smem_u32;
using tc::sw128_desc;
using tc::tma_load_2d;
using tc::tmem_alloc;
using tc::tmem_dealloc;
using tc::tmem_ld16_nowait;
using tc::tmem_wait16;

constexpr int BM = 128;
constexpr int THREADS = 448;
constexpr int SPLIT_W0 = 2, EPI_W0 = 6;
constexpr int MAX_STAGES = 4;

struct Params {
  int tf32;                    // 1: fp32 operands (3xTF32), 0: bf16
  int a_mn, b_mn;              // 1: the operand's M (A) / N (B) index is the contiguous one
  int64_t M_max; const int32_t* M_dev;
  int N;
  int64_t K_max; const int32_t* K_dev;
  int BN, n_tiles, k_splits, kb_per_split;
  int stages;
  uint32_t a_bytes, b_bytes;   // one precision plane of a stage's A / B tile
  uint32_t a_box, b_box;       // bytes of one M/N-major TMA box (64 or 32 MN x BK)
  int at;                      // elements per 128-byte swizzle atom (32 fp32, 64 bf16)
  const float* bias; int relu; int accumulate;
  float* C; int64_t ldc; int vec;
  float* const* out_base; const int32_t* out_rank; const int32_t* out_row;
  int ones_col; float* ones_out;
  int tmem_cols;
  uint16_t* Yb; int64_t yb_pitch;   // bf16 rows instead of C (hidden activations, reading R11)
};

__device__ __forceinline__ void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc)
      : "memory");
}

// kind::f16 / kind::tf32 instruction descriptor: D fp32, A/B bf16 (1) or tf32 (2).
__host__ __device__ __forceinline__ uint32_t idesc_of(int tf32, int M, int N, int a_mn, int b_mn) {
  const uint32_t f = tf32 ? 2u : 1u;
  return (1u << 4) | (f << 7) | (f << 10) | (uint32_t(a_mn) << 15) | (uint32_t(b_mn) << 16) |
         (uint32_t(N >> 3) << 17) | (uint32_t(M >> 4) << 24);
}

// SW128 descriptors of the kk-th MMA K-slice of a tile: K-major rows of 128 B (slice =
// 32 B further); M/N-major boxes of one swizzle atom of M/N x BK rows of K, `box` bytes
// apart (LBO), 8-row groups 1 KB apart (SBO), slice = mma_k rows of 128 B further.
__device__ __forceinline__ uint64_t desc_of(uint32_t base, int mn_major, int kk, int mma_k, uint32_t box) {
  return mn_major ? sw128_desc(base + uint32_t(kk * mma_k * 128), box, 1024) : sw128_desc(base + uint32_t(kk * 32), 16, 1024);
}

// Tile t -> (m tile, n tile, k split) and its k-block range [kb0, kb1).
struct TileInfo { int64_t mt; int nt, ks; int64_t kb0, kb1; };
__device__ __forceinline__ TileInfo tile_info(const Params& p, int64_t t, int64_t nkb) {
  TileInfo ti;
  ti.ks = int(t % p.k_splits);
  const int64_t r = t / p.k_splits;
  ti.nt = int(r % p.n_tiles);
  ti.mt = r / p.n_tiles;
  ti.kb0 = int64_t(ti.ks) * p.kb_per_split;
  ti.kb1 = std::min<int64_t>(nkb, ti.kb0 + p.kb_per_split);
  return ti;
}

// hi / lo split of one K-major fp32 operand tile in place (rows of 128 B = 32 K;
// SW128 permutes 16-byte chunks inside a row, so a word keeps its tile position),
// zeroing every word whose K index is >= K (a device-counted K: stale rows of a reused
// buffer).  x_hi = RN_tf32(x), x_lo = x - x_hi (exact).
__device__ __forceinline__ void split_k_major(uint8_t* hi, uint8_t* lo, uint32_t bytes, int64_t k0, int64_t K,
                                              int tid, int nthreads) {
  for (uint32_t off = uint32_t(tid) * 16; off < bytes; off += uint32_t(nthreads) * 16) {
    const float4 x = *reinterpret_cast<const float4*>(hi + off);
    const uint32_t row = off >> 7, chunk = (off >> 4) & 7;
    const int64_t kq = k0 + int64_t((chunk ^ (row & 7)) << 2);
    const float w[4] = {x.x, x.y, x.z, x.w};
    float h[4], l[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float v = kq + j < K ? w[j] : 0.f;
      uint32_t hb;
      asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(hb) : "f"(v));
      h[j] = __uint_as_float(hb);
      l[j] = v - h[j];
    }
    *reinterpret_cast<float4*>(hi + off) = make_float4(h[0], h[1], h[2], h[3]);
    *reinterpret_cast<float4*>(lo + off) = make_float4(l[0], l[1], l[2], l[3]);
  }
}

// The same split of an M/N-major fp32 tile (R <= 128 M/N rows x 32 K, TMA boxes of 32
// M/N x 32 K rows, 4 KB apart), TRANSPOSED on the way into the K-major SW128 form the
// kind::tf32 MMA reads (the M/N-major 32-bit canonical layout differs from 16-bit
// types'; one K-major layout serves every operand).  All 128 splitter threads read
// their chunks into registers, sync, then write hi (in place) and lo.
__device__ __forceinline__ void split_mn_major(uint8_t* hi, uint8_t* lo, int R, int64_t k0, int64_t K, int tid) {
  float4 v[8];
  const int nchunks = R * 8;            // 16-byte chunks of the tile
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int q = tid + i * 128;
    if (q < nchunks) v[i] = *reinterpret_cast<const float4*>(hi + q * 16);
  }
  asm volatile("bar.sync 1, 128;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int q = tid + i * 128;
    if (q >= nchunks) break;
    // source chunk q: box j, K row k, stored chunk sc -> logical chunk c16 = sc ^ (k & 7)
    const int j = q >> 8, k = (q >> 3) & 31, sc = q & 7, c16 = sc ^ (k & 7);
    const float w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
    const bool keep = k0 + k < K;
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int mn = j * 32 + c16 * 4 + e;
      const uint32_t dst = uint32_t(mn) * 128 + (uint32_t(((k >> 2) ^ (mn & 7))) << 4) + uint32_t(k & 3) * 4;
      const float x = keep ? w[e] : 0.f;
      uint32_t hb;
      asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(hb) : "f"(x));
      *reinterpret_cast<float*>(hi + dst) = __uint_as_float(hb);
      *reinterpret_cast<float*>(lo + dst) = x - __uint_as_float(hb);
    }
  }
  asm volatile("bar.sync 1, 128;" ::: "memory");
}

__global__ void __launch_bounds__(THREADS, 1)
    gen_gemm_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB, Params p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t plane = p.a_bytes + p.b_bytes;                   // one precision plane of a stage
  const uint32_t stage_bytes = plane * (p.tf32 ? 2u : 1u);        // [hi A | hi B | lo A | lo B]
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + size_t(p.stages) * stage_bytes);
  uint64_t* full = bars;                       // [MAX_STAGES] TMA landed
  uint64_t* conv = bars + MAX_STAGES;          // [MAX_STAGES] split done (fp32)
  uint64_t* empty = bars + 2 * MAX_STAGES;     // [MAX_STAGES] MMAs of the stage done
  uint64_t* tfull = bars + 3 * MAX_STAGES;     // [2]
  uint64_t* tempty = tfull + 2;                // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = lane_id();
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < MAX_STAGES; ++s) { mbar_init(full + s, 1); mbar_init(conv + s, 128); mbar_init(empty + s, 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(tfull + a, 1); mbar_init(tempty + a, 256); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapB)) : "memory");
  }
  if (warp == 1) tmem_alloc(tmem_slot, uint32_t(p.tmem_cols));
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem_base = *tmem_slot;
  pdl_wait();
  pdl_launch();
  const int64_t M = p.M_dev ? std::min<int64_t>(p.M_max, int64_t(*p.M_dev)) : p.M_max;
  const int64_t K = p.K_dev ? std::min<int64_t>(p.K_max, int64_t(*p.K_dev)) : p.K_max;
  const int BK = p.at;
  const int64_t nkb = ceil_div(K, BK);
  const int64_t ntiles = ceil_div(M, BM) * p.n_tiles * p.k_splits;
  const int mma_k = p.tf32 ? 8 : 16;

  if (warp == 0) {
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const TileInfo ti = tile_info(p, t, nkb);
        for (int64_t kb = ti.kb0; kb < ti.kb1; ++kb) {
          mbar_wait(empty + s, ph ^ 1);
          mbar_expect_tx(full + s, plane);
          uint8_t* sa = smem + size_t(s) * stage_bytes;
          uint8_t* sb = sa + p.a_bytes;
          const int k = int(kb * BK);
          if (p.a_mn) {
            for (int j = 0; j < BM / p.at; ++j) tma_load_2d(sa + j * p.a_box, &mapA, full + s, int(ti.mt * BM) + j * p.at, k);
          } else {
            tma_load_2d(sa, &mapA, full + s, k, int(ti.mt * BM));
          }
          if (p.b_mn) {
            for (int j = 0; j < p.BN / p.at; ++j) tma_load_2d(sb + j * p.b_box, &mapB, full + s, ti.nt * p.BN + j * p.at, k);
          } else {
            tma_load_2d(sb, &mapB, full + s, k, ti.nt * p.BN);
          }
          if (++s == p.stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    int s = 0, acc = 0;
    uint32_t ph = 0, aph = 0;
    // tf32 operands are K-major in shared memory after the split (split_mn_major)
    const int am = p.tf32 ? 0 : p.a_mn, bm = p.tf32 ? 0 : p.b_mn;
    const uint32_t idesc = idesc_of(p.tf32, BM, p.BN, am, bm);
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const TileInfo ti = tile_info(p, t, nkb);
      if (ti.kb0 >= ti.kb1) continue;
      mbar_wait(tempty + acc, aph ^ 1);
      fence_after();
      const uint32_t d = tmem_base + uint32_t(acc * p.BN);
      for (int64_t kb = ti.kb0; kb < ti.kb1; ++kb) {
        mbar_wait((p.tf32 ? conv : full) + s, ph);
        fence_after();
        if (lane == 0) {
          const uint32_t a_hi = smem_u32(smem + size_t(s) * stage_bytes), b_hi = a_hi + p.a_bytes;
          const uint32_t a_lo = a_hi + plane, b_lo = b_hi + plane;
          for (int kk = 0; kk < BK / mma_k; ++kk) {
            const uint32_t first = (kb > ti.kb0 || kk) ? 1u : 0u;
            const uint64_t dah = desc_of(a_hi, am, kk, mma_k, p.a_box), dbh = desc_of(b_hi, bm, kk, mma_k, p.b_box);
            if (p.tf32) {
              mma_tf32(d, dah, dbh, idesc, first);
              mma_tf32(d, desc_of(a_lo, am, kk, mma_k, p.a_box), dbh, idesc, 1u);
              mma_tf32(d, dah, desc_of(b_lo, bm, kk, mma_k, p.b_box), idesc, 1u);
            } else {
              tc::mma_bf16(d, dah, dbh, idesc, first);
            }
          }
          mma_commit(empty + s);
        }
        __syncwarp();
        if (++s == p.stages) { s = 0; ph ^= 1; }
      }
      if (lane == 0) mma_commit(tfull + acc);
      __syncwarp();
      if (++acc == 2) { acc = 0; aph ^= 1; }
    }
  } else if (warp < EPI_W0) {
    if (p.tf32) {
      const int tid = threadIdx.x - SPLIT_W0 * 32;
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const TileInfo ti = tile_info(p, t, nkb);
        for (int64_t kb = ti.kb0; kb < ti.kb1; ++kb) {
          mbar_wait(full + s, ph);
          uint8_t* sa = smem + size_t(s) * stage_bytes;
          if (p.a_mn) split_mn_major(sa, sa + plane, BM, kb * BK, K, tid);
          else split_k_major(sa, sa + plane, p.a_bytes, kb * BK, K, tid, 128);
          if (p.b_mn) split_mn_major(sa + p.a_bytes, sa + plane + p.a_bytes, p.BN, kb * BK, K, tid);
          else split_k_major(sa + p.a_bytes, sa + plane + p.a_bytes, p.b_bytes, kb * BK, K, tid, 128);
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic writes -> tensor-core reads
          mbar_arrive(conv + s);
          if (++s == p.stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else {
    const int q = warp & 3, h = (warp - EPI_W0) >> 2;
    int acc = 0;
    uint32_t aph = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const TileInfo ti = tile_info(p, t, nkb);
      if (ti.kb0 >= ti.kb1) continue;
      mbar_wait(tfull + acc, aph);
      fence_after();
      const int64_t m = ti.mt * BM + q * 32 + lane;
      float* row = nullptr;
      if (m < M)
        row = p.Yb ? reinterpret_cast<float*>(p.Yb + m * p.yb_pitch)
                   : (p.out_rank ? p.out_base[p.out_rank[m]] + int64_t(p.out_row[m]) * p.ldc : p.C + m * p.ldc);
      const bool add_bias = p.bias && ti.ks == 0;
      const uint32_t tbase = tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * p.BN);
      uint32_t r[16], rn[16];
      if (16 * h < p.BN) tmem_ld16_nowait(tbase + uint32_t(16 * h), r);
      if (16 * h < p.BN) tmem_wait16(r);
      for (int c = 16 * h; c < p.BN; c += 32) {
        const bool more = c + 32 < p.BN;
        if (more) tmem_ld16_nowait(tbase + uint32_t(c + 32), rn);
        const int n0 = ti.nt * p.BN + c;
        if (row) {
          float v[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            v[j] = __uint_as_float(r[j]);
            if (add_bias && n0 + j < p.N) v[j] += p.bias[n0 + j];
            if (p.relu) v[j] = fmaxf(v[j], 0.f);
          }
          const bool plain = p.vec && n0 + 16 <= p.N && !(p.ones_col >= n0 && p.ones_col < n0 + 16);
          if (p.Yb) {
            uint16_t* d = reinterpret_cast<uint16_t*>(row) + n0;
            if (n0 + 16 <= p.N && (reinterpret_cast<uintptr_t>(d) & 31) == 0) {   // one 32-byte sector store
              st_v8(d, pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                    pack_bf16x2(v[6], v[7]), pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]),
                    pack_bf16x2(v[12], v[13]), pack_bf16x2(v[14], v[15]));
            } else if (n0 + 16 <= p.N) {
              reinterpret_cast<uint4*>(d)[0] = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
                                                          pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
              reinterpret_cast<uint4*>(d)[1] = make_uint4(pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]),
                                                          pack_bf16x2(v[12], v[13]), pack_bf16x2(v[14], v[15]));
            } else {
              for (int j = 0; j < 16 && n0 + j < p.N; ++j) d[j] = bf16_bits(v[j]);
            }
          } else if (plain) {
            float* d = row + n0;
            if (!p.accumulate && (reinterpret_cast<uintptr_t>(d) & 31) == 0) {   // whole 32-byte sectors
#pragma unroll
              for (int j = 0; j < 16; j += 8)
                st_v8(d + j, __float_as_uint(v[j]), __float_as_uint(v[j + 1]), __float_as_uint(v[j + 2]),
                      __float_as_uint(v[j + 3]), __float_as_uint(v[j + 4]), __float_as_uint(v[j + 5]),
                      __float_as_uint(v[j + 6]), __float_as_uint(v[j + 7]));
            } else {
#pragma unroll
              for (int j = 0; j < 16; j += 4) {
                if (p.accumulate) red_add_v4(d + j, v[j], v[j + 1], v[j + 2], v[j + 3]);
                else *reinterpret_cast<float4*>(d + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
              }
            }
          } else {
#pragma unroll
            for (int j = 0; j < 16; ++j) {
              const int n = n0 + j;
              if (n >= p.N) break;
              if (n == p.ones_col) {
                if (p.ones_out) atomicAdd(p.ones_out + m, v[j]);
              } else if (p.accumulate) {
                atomicAdd(row + n, v[j]);
              } else {
                row[n] = v[j];
              }
            }
          }
        }
        if (more) {
          tmem_wait16(rn);
#pragma unroll
          for (int j = 0; j < 16; ++j) r[j] = rn[j];
        }
      }
      fence_before();
      mbar_arrive(tempty + acc);
      if (++acc == 2) { acc = 0; aph ^= 1; }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem_base, uint32_t(p.tmem_cols));
  }
}

// 2-D map of a row-major [rows x cols] matrix (cols contiguous, `pitch` elements per row)
// of fp32 or bf16, SW128, box {box_cols, box_rows}, zero fill out of bounds.
static bool make_map2(CUtensorMap* m, const void* base, bool f32, int64_t cols, int64_t rows, int64_t pitch,
                      int box_cols, int box_rows) {
  auto fn = tc::encode_fn();
  if (!fn) return false;
  const int e = f32 ? 4 : 2;
  cuuint64_t dims[2] = {cuuint64_t(cols), cuuint64_t(std::max<int64_t>(rows, 1))};
  cuuint64_t strides[1] = {cuuint64_t(pitch * e)};
  cuuint32_t box[2] = {cuuint32_t(box_cols), cuuint32_t(box_rows)};
  cuuint32_t estr[2] = {1, 1};
  return fn(m, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims,
            strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace tcg

// The operand is usable by TMA: one unit stride, the other a 16-byte multiple, base
// 16-byte aligned.
static bool tma_ok(const void* base, int e, int64_t s0, int64_t s1) {
  if (reinterpret_cast<uintptr_t>(base) & 15) return false;
  const int64_t other = s0 == 1 ? s1 : (s1 == 1 ? s0 : -1);
  return other > 0 && (other * e) % 16 == 0;
}

int tc_gen_supported(const SimtGemmArgs& a) {
  if (a.a_t != a.b_t) return 0;
  const int e = a.a_t == kF32 ? 4 : 2;
  if (!tma_ok(a.A, e, a.sak, a.sam) || !tma_ok(a.B, e, a.sbk, a.sbn)) return 0;
  if (a.relu && a.accumulate) return 0;
  if (a.N < 1 || a.M < 1 || a.K < 1) return 0;
  return 1;
}

// The tensor-core path of launch_simt_gemm's contract (kernels.h SimtGemmArgs).
cudaError_t launch_tc_gen_gemm(const SimtGemmArgs& a, int ones_col, float* ones_out, cudaStream_t st) {
  using namespace tcg;
  if (!tc_gen_supported(a)) return cudaErrorInvalidValue;
  const bool f32 = a.a_t == kF32;
  const int e = f32 ? 4 : 2, at = 128 / e, BK = at;
  Params p{};
  p.tf32 = f32 ? 1 : 0;
  p.a_mn = a.sam == 1 && a.sak != 1 ? 1 : 0;
  p.b_mn = a.sbn == 1 && a.sbk != 1 ? 1 : 0;
  p.M_max = a.M; p.M_dev = a.M_dev; p.N = a.N; p.K_max = a.K; p.K_dev = a.K_dev;
  p.at = at;
  // N in slices of <= 256 columns (multiples of 16; M/N-major B: of the 128-byte atom)
  const int nq = p.b_mn ? at : 16;
  p.BN = int(std::min<int64_t>((f32 && p.b_mn) ? 128 : 256, round_up(a.N, nq)));
  p.BN = int(round_up(p.BN, 16));
  p.n_tiles = int(ceil_div(a.N, p.BN));
  p.a_bytes = uint32_t(BM) * 128;
  p.b_bytes = uint32_t(p.BN) * 128;
  p.a_box = uint32_t(at) * BK * e;          // = 128 B x BK rows
  p.b_box = p.a_box;
  const uint32_t stage = (p.a_bytes + p.b_bytes) * (f32 ? 2u : 1u);
  p.stages = int(std::min<int64_t>(MAX_STAGES, (200 * 1024) / stage));
  if (p.stages < 2) return cudaErrorInvalidValue;
  int cols = 32;
  while (cols < 2 * p.BN) cols <<= 1;
  p.tmem_cols = cols;
  // split-K: only with an accumulating epilogue (the caller zeroed C); enough tiles
  // for every SM
  const int64_t nkb = ceil_div(a.K, BK);
  const int64_t mn_tiles = ceil_div(a.M, BM) * p.n_tiles;
  int ks = 1;
  if (a.accumulate) ks = int(std::max<int64_t>(1, std::min<int64_t>(nkb, num_sms() / std::max<int64_t>(1, mn_tiles))));
  p.k_splits = ks;
  p.kb_per_split = int(ceil_div(nkb, ks));
  p.bias = a.bias; p.relu = a.relu; p.accumulate = a.accumulate;
  p.C = a.C; p.ldc = a.ldc;
  p.vec = (a.ldc % 4 == 0) && !(reinterpret_cast<uintptr_t>(a.C) & 15) ? 1 : 0;
  if (a.out_rank) p.vec = a.ldc % 4 == 0 ? 1 : 0;   // peer buffers: 256-B aligned allocations
  p.out_base = a.out_base; p.out_rank = a.out_rank; p.out_row = a.out_row;
  p.ones_col = ones_col; p.ones_out = ones_out;
  p.Yb = a.Cb; p.yb_pitch = a.ldcb;
  if (a.Cb && (a.out_rank || a.accumulate || (a.ldcb % 8) || (reinterpret_cast<uintptr_t>(a.Cb) & 15)))
    return cudaErrorInvalidValue;
  CUtensorMap ma, mb;
  // A(m, k) = A[m * sam + k * sak]
  bool ok = p.a_mn ? make_map2(&ma, a.A, f32, a.M, a.K, a.sak, at, BK) : make_map2(&ma, a.A, f32, a.K, a.M, a.sam, BK, BM);
  ok = ok && (p.b_mn ? make_map2(&mb, a.B, f32, a.N, a.K, a.sbk, at, BK)
                     : make_map2(&mb, a.B, f32, a.K, a.N, a.sbn, BK, p.BN));
  if (!ok) return cudaErrorInvalidValue;
  const size_t smem = 1024 + size_t(p.stages) * stage + 256;
  static std::once_flag once;
  std::call_once(once, [] { cudaFuncSetAttribute(gen_gemm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024); });
  const int64_t tiles = mn_tiles * ks;
  const int grid = int(std::max<int64_t>(1, std::min<int64_t>(tiles, num_sms())));
  launch_pdl(gen_gemm_kernel, dim3(grid), dim3(THREADS), smem, st, ma, mb, p);
  return cudaGetLastError();
}

}  // namespace apt

// Self-test of the general tcgen05 GEMM (apt.h): C = A B (+ bias) for operands of the
// given type and majorness, M x N x K, optionally split-K accumulating into a zeroed C,
// against an fp64 host product of the same (rounded) operands.  Returns the largest
// |C - ref| / (sum_k |A||B| + |bias|) over the elements (the error relative to the
// magnitude of the terms), or < 0 on failure.  Uses the current device; syncs.
extern "C" double apt_selftest_gemm(int f32, int a_mn, int b_mn, int64_t M, int N, int64_t K, int accumulate) {
  using namespace apt;
  if (M < 1 || N < 1 || K < 1) return -1;
  const int e = f32 ? 4 : 2;
  const int64_t pa = a_mn ? round_up(M, 8) : round_up(K, 8), ra = a_mn ? K : M;   // rows x pitch of A
  const int64_t pb = b_mn ? round_up(N, 8) : round_up(K, 8), rb = b_mn ? K : N;
  std::vector<float> A(ra * pa, 0.f), B(rb * pb, 0.f), bias(N);
  uint32_t st = 12345u;
  auto rnd = [&]() { st = st * 1664525u + 1013904223u; return (int32_t(st >> 8) - (1 << 23)) / float(1 << 23); };
  auto rbf = [&](float x) {   // bf16 RNE
    uint32_t b; memcpy(&b, &x, 4); b = (b + 0x7FFFu + ((b >> 16) & 1u)) & 0xFFFF0000u; float y; memcpy(&y, &b, 4); return y;
  };
  for (auto& x : A) x = f32 ? rnd() : rbf(rnd());
  for (auto& x : B) x = f32 ? rnd() : rbf(rnd());
  for (auto& x : bias) x = rnd();
  auto a_at = [&](int64_t m, int64_t k) { return double(a_mn ? A[k * pa + m] : A[m * pa + k]); };
  auto b_at = [&](int64_t k, int64_t n) { return double(b_mn ? B[k * pb + n] : B[n * pb + k]); };
  std::vector<uint16_t> Ah, Bh;
  auto to_bits = [](const std::vector<float>& v, std::vector<uint16_t>& o) {
    o.resize(v.size());
    for (size_t i = 0; i < v.size(); ++i) { uint32_t b; memcpy(&b, &v[i], 4); o[i] = uint16_t(b >> 16); }
  };
  void *dA = nullptr, *dB = nullptr;
  float *dC = nullptr, *dbias = nullptr;
  const int64_t ldc = round_up(N, 4);
  if (cudaMalloc(&dA, A.size() * e) || cudaMalloc(&dB, B.size() * e) || cudaMalloc(&dC, M * ldc * 4) ||
      cudaMalloc(&dbias, N * 4))
    return -2;
  if (f32) {
    cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
  } else {
    to_bits(A, Ah); to_bits(B, Bh);
    cudaMemcpy(dA, Ah.data(), Ah.size() * 2, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, Bh.data(), Bh.size() * 2, cudaMemcpyHostToDevice);
  }
  cudaMemcpy(dbias, bias.data(), N * 4, cudaMemcpyHostToDevice);
  cudaMemset(dC, 0, M * ldc * 4);
  SimtGemmArgs g{};
  g.A = dA; g.a_t = f32 ? kF32 : kBF16; g.sam = a_mn ? 1 : pa; g.sak = a_mn ? pa : 1;
  g.B = dB; g.b_t = g.a_t; g.sbk = b_mn ? pb : 1; g.sbn = b_mn ? 1 : pb;
  g.C = dC; g.ldc = ldc; g.bias = dbias; g.M = M; g.N = N; g.K = K; g.accumulate = accumulate;
  cudaError_t err = launch_tc_gen_gemm(g, -1, nullptr, 0);
  if (err == cudaSuccess) err = cudaDeviceSynchronize();
  std::vector<float> C(M * ldc);
  cudaMemcpy(C.data(), dC, C.size() * 4, cudaMemcpyDeviceToHost);
  cudaFree(dA); cudaFree(dB); cudaFree(dC); cudaFree(dbias);
  if (err != cudaSuccess) return -3;
  double worst = 0;
  for (int64_t m = 0; m < M; ++m)
    for (int n = 0; n < N; ++n) {
      double ref = bias[n], mag = std::fabs(bias[n]);
      for (int64_t k = 0; k < K; ++k) {
        const double t = a_at(m, k) * b_at(k, n);
        ref += t;
        mag += std::fabs(t);
      }
      worst = std::max(worst, std::fabs(C[m * ldc + n] - ref) / std::max(mag, 1e-30));
    }
  return worst;
}
