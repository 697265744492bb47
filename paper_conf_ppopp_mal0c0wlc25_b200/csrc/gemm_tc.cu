// gemm_tc.cu -- the dense contractions of the step on the 5th-generation tensor
// cores (tcgen05, bf16 operands, fp32 accumulation in TMEM):
//
//   S8   projection      Y  = Z W^T + b (ReLU)     (Eq. 1; Fig. 5
//                                                  "dense tensor multiplication")
//   S10  input gradient  dZ = G W                  (backward of the projection)
//   S11  weight gradient dW = G^T Z, db = G^T 1    (split over the rows)
//
// sm_100a design:
//  * rowtile kernel (projection, dZ): persistent CTAs (grid <= #SMs), one
//    128-row M tile per iteration.  The B operand (W, <= 256 x 256 bf16) is
//    TMA-loaded once per CTA and stays resident in shared memory; A tiles
//    (128 x 64 bf16, 128-B swizzle) stream through a 4-stage mbarrier ring.
//    Warp 0 = TMA producer, warp 1 = TMEM allocator + single-thread MMA issuer
//    (M=128, N=BN, K=16 per instruction) with double-buffered accumulators so
//    the epilogue of tile i overlaps the MMAs of tile i+1, warps 2..5 =
//    epilogue (tcgen05.ld 32x32b -> +bias -> ReLU -> fp32 stores; a row may be
//    routed to another rank's buffer: the peer-store epilogue of the strategies).
//  * wgrad kernel (dW, db): the reduction runs over the sampled rows, so both
//    operands are MN-major in memory (G [rows x d_out], Z [rows x d_in]); grid =
//    (row splits) x (128-wide d_out tiles), each CTA accumulates its row range in
//    TMEM (N up to 512 columns: d_in plus the all-ones column of Z that turns
//    the bias gradient into one more output column), then adds it into dW/db
//    with 16-byte vector reductions.
// Operand layouts (CUTLASS canonical forms, uint128 units, SW128):
//  * K-major : ((8,m),(8,2)) : ((8,SBO),(1,...)), rows of 128 B, SBO = 1024 B;
//              the k-th K=16 slice starts 32 B further.
//  * MN-major: ((8,n),(8,k)) : ((1,LBO),(8,SBO)); one TMA box = 64 MN x 64 K =
//              8 KB, boxes of consecutive MN blocks 8 KB apart (LBO = 8192),
//              8-row K groups 1024 B apart (SBO); the k-th K=16 slice starts
//              2048 B further.
// The projection is HBM-bound (AI <= 114 FLOP/B < ridge ~250), so the design
// goal is streaming A and the outputs at full bandwidth, not MMA throughput.
#include "common.cuh"
#include "kernels.h"
#include "tc_common.cuh"
#include <cuda.h>
#include <cudaTypedefs.h>
#include <algorithm>
#include <cstdlib>
#include <mutex>

namespace apt {

namespace tc {

// ------------------------------------------------------------ row-tile kernel
struct RowParams {
  int64_t M_max;
  const int32_t* M_dev;
  int N, BN, nkb, tmem_cols, b_mn;
  int stages;               // A ring depth (<= STAGES)
  int nacc;                 // TMEM accumulator buffers (2: epilogue overlaps the next tile's MMAs)
  uint32_t b_kb_bytes;      // bytes of one resident B k-block
  const float* bias;
  int relu;
  float* Y;
  int64_t y_pitch;
  float* const* out_base;
  const int32_t* out_rank;
  const int32_t* out_row;
  int accumulate;
  int n_split;              // CTAs share an M tile: CTA b computes columns [(b % n_split) * BN, +BN)
  uint16_t* mask;           // optional ReLU bit mask [M x mask_pitch] (16 columns per word)
  int64_t mask_pitch;
  int mask_direct;          // the mask comes from the direct (bf16-row) epilogue
  const int32_t* row_div;   // optional: divide row m by indptr[m+1] - indptr[m] (RN)
  uint16_t* Yb;             // optional bf16 output instead of Y (not with routing / accumulation)
  int64_t yb_pitch;
  int b_early;              // B (W) is not written by the preceding kernel: load it before the PDL wait
  int staged;               // force the staged epilogue for plain rows too (APT_EPI_STAGED=1, A/B)
  int tma_store;            // bf16 rows, BN == 128: each warp's 32 x 64 block leaves through a TMA store
};

__global__ void __launch_bounds__(ROW_THREADS, 1)
    rowtile_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                   const __grid_constant__ CUtensorMap mapY, RowParams p) {
  // Programmatic dependent launch: barrier init, TMEM allocation, tensor-map prefetch
  // and (b_early) the resident B load run before griddepcontrol.wait, i.e. while the
  // preceding kernel of the step drains; everything that reads its outputs (the row
  // count, A) or writes global memory comes after the wait.
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);   // 1 KB aligned, still __shared__
  uint8_t* smem_a = smem;                                        // stages x 16 KB
  uint8_t* smem_b = smem + p.stages * A_STAGE_BYTES;             // nkb x b_kb_bytes
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_b + size_t(p.nkb) * p.b_kb_bytes);
  uint64_t* full = bars;                  // [STAGES]
  uint64_t* empty = bars + STAGES;        // [STAGES]
  uint64_t* bfull = bars + 2 * STAGES;    // [1]
  uint64_t* tfull = bfull + 1;            // [2]
  uint64_t* tempty = tfull + 2;           // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  float* sbias = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(bars) + 128);           // [<= 256]
  float* stg_all = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(bars) + 128 + 1024);   // [8][32][17]
  // TMA-store staging (tma_store): per epilogue warp two 4 KB buffers of 32 rows x 128 B,
  // 1 KB aligned (the 128-byte swizzle of the output map)
  uint8_t* ystage = reinterpret_cast<uint8_t*>(
      (reinterpret_cast<uintptr_t>(stg_all + 8 * 32 * 17) + 1023) & ~uintptr_t(1023));

  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int n0 = int(blockIdx.x % p.n_split) * p.BN;              // this CTA's column slice
  const int64_t t0 = blockIdx.x / p.n_split, tstride = gridDim.x / p.n_split;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    mbar_init(bfull, 1);   // (barrier slots are laid out for the maximum STAGES)
    for (int a = 0; a < 2; ++a) { mbar_init(tfull + a, 1); mbar_init(tempty + a, 256); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapB)) : "memory");
    if (p.tma_store) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapY)) : "memory");
  }
  if (warp == 1) tmem_alloc(tmem_slot, uint32_t(p.tmem_cols));
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem_base = *tmem_slot;
  // resident B (this CTA's column slice): W does not depend on the preceding kernel when
  // the caller says so (b_early), so its load overlaps that kernel's tail
  auto load_b = [&]() {
    mbar_expect_tx(bfull, uint32_t(p.nkb) * p.b_kb_bytes);
    const int nb = int(ceil_div(p.BN, 64));
    for (int kb = 0; kb < p.nkb; ++kb) {
      uint8_t* dst = smem_b + size_t(kb) * p.b_kb_bytes;
      if (p.b_mn) {
        for (int j = 0; j < nb; ++j) tma_load_2d(dst + j * MNBLK, &mapB, bfull, n0 + j * 64, kb * BK);
      } else {
        tma_load_2d(dst, &mapB, bfull, kb * BK, n0);
      }
    }
  };
  if (p.b_early && warp == 0 && lane == 0) load_b();
  pdl_wait();
  pdl_launch();
  const int64_t M = std::min<int64_t>(p.M_max, int64_t(*p.M_dev));
  const int64_t ntiles = ceil_div(M, BM);

  if (warp == 0) {
    if (lane == 0 && p.b_early && ntiles <= t0) mbar_wait(bfull, 0);   // no tile: let B land before exit
    if (lane == 0 && ntiles > t0) {
      // ---- TMA producer: resident B (unless loaded early), then the A ring
      if (!p.b_early) load_b();
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = t0; t < ntiles; t += tstride) {
        for (int kb = 0; kb < p.nkb; ++kb) {
          mbar_wait(empty + s, ph ^ 1);
          mbar_expect_tx(full + s, A_STAGE_BYTES);
          tma_load_2d(smem_a + s * A_STAGE_BYTES, &mapA, full + s, kb * BK, int(t * BM));
          if (++s == p.stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ---- MMA issuer (one thread)
    if (ntiles > t0) {
      const uint32_t idesc = idesc_bf16(BM, p.BN, 0, p.b_mn);
      mbar_wait(bfull, 0);
      fence_after();
      int s = 0;
      uint32_t ph = 0;
      int acc = 0;
      uint32_t aph = 0;
      for (int64_t t = t0; t < ntiles; t += tstride) {
        mbar_wait(tempty + acc, aph ^ 1);
        fence_after();
        const uint32_t d = tmem_base + uint32_t(acc * p.BN);
        for (int kb = 0; kb < p.nkb; ++kb) {
          mbar_wait(full + s, ph);
          fence_after();
          if (lane == 0) {
            const uint32_t a0 = smem_u32(smem_a + s * A_STAGE_BYTES);
            const uint32_t b0 = smem_u32(smem_b + size_t(kb) * p.b_kb_bytes);
#pragma unroll
            for (int kk = 0; kk < BK / 16; ++kk)
              mma_bf16(d, desc_k(a0, kk), p.b_mn ? desc_mn(b0, kk) : desc_k(b0, kk), idesc, (kb | kk) != 0);
            mma_commit(empty + s);            // frees the smem stage when these MMAs finish
          }
          __syncwarp();
          if (++s == p.stages) { s = 0; ph ^= 1; }
        }
        if (lane == 0) mma_commit(tfull + acc);   // accumulator ready for the epilogue
        __syncwarp();
        if (++acc == p.nacc) { acc = 0; aph ^= 1; }
      }
    }
  } else {
    // ---- epilogue warps 2..9: TMEM lane quarter q = warp % 4 (hardware rule), column
    // half h: the warp takes every other 16-column chunk.  A chunk of the warp's 32
    // rows is staged in shared memory (row stride 17 floats: conflict-free writes) and
    // written back row-contiguously: 4 lanes cover one 64-B row segment, so a store
    // instruction moves 8 segments instead of 32 scattered 16-B pieces.  Eight
    // warps keep twice the independent TMEM-load -> store chains in flight.  The
    // bias slice sits in shared memory (loaded once per CTA) and the next chunk's TMEM
    // load is issued before the current chunk is processed, so a chunk's critical path
    // is shared-memory latency, not a global bias load and a TMEM round trip.
    const int q = warp & 3, h = (warp - 2) >> 2;
    // staged: 0 direct for every plain output, 1 never (A/B), 2 only for bf16 rows
    // (bf16 rows may also emit their ReLU bit mask from the direct path: mask_direct)
    const bool direct = !p.out_rank && !p.accumulate && (!p.mask || p.mask_direct) &&
                        (p.staged == 0 || (p.staged == 2 && p.Yb));
    float* stg = stg_all + (warp - 2) * 32 * 17;
    const int rsub = lane >> 2, cq = (lane & 3) * 4;
    // this CTA's bias slice (zero past N or without bias), shared by the 8 epilogue warps
    for (int j = threadIdx.x - 64; j < p.BN; j += 256) sbias[j] = (p.bias && n0 + j < p.N) ? p.bias[n0 + j] : 0.f;
    asm volatile("bar.sync 1, 256;" ::: "memory");
    int acc = 0;
    uint32_t aph = 0;
    int ybuf = 0;
    for (int64_t t = t0; t < ntiles; t += tstride) {
      mbar_wait(tfull + acc, aph);
      fence_after();
      // own row (= TMEM lane) destination; shuffled to the lanes that store it
      const int64_t m_own = t * BM + q * 32 + lane;
      float* own = nullptr;
      if (m_own < M) {
        if (p.Yb) own = reinterpret_cast<float*>(p.Yb + m_own * p.yb_pitch);   // bf16 row (reading R11)
        else if (p.out_rank) own = p.out_base[p.out_rank[m_own]] + int64_t(p.out_row[m_own]) * p.y_pitch;
        else own = p.Y + m_own * p.y_pitch;
      }
      float own_deg = 0.f;
      if (p.row_div && m_own < M) own_deg = float(p.row_div[m_own + 1] - p.row_div[m_own]);
      const float own_rdeg = own_deg > 0.f ? __frcp_rn(own_deg) : 0.f;
      const uint32_t tbase = tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * p.BN);
      if (direct) {
        // Direct path (plain rows: no routing, reduction or mask): the lane owns its row
        // (its TMEM lane) and writes straight from registers -- no staging, shuffles or
        // per-element branches.  The warp owns a contiguous half of the tile's 16-column
        // chunks and loads up to four of them (64 columns) before ONE wait, so a lane
        // writes up to 128 contiguous bytes of its row per group and the TMEM round trip
        // is paid once per group, not per chunk (ncu: the one-chunk-in-flight loop was
        // latency-bound at ~10 cycles per issued instruction with 2 warps per scheduler).
        const int nch = p.BN / 16, half = (nch + 1) / 2;
        const int cb0 = h * half, cb1 = min(nch, cb0 + half);
        // tma_store: the warp's 32 rows x 64 columns go through a shared-memory box in the
        // output map's 128-byte swizzle (row r's 16-byte unit u at (u ^ (r & 7)) * 16: 8
        // consecutive rows cover all banks) and leave as ONE bulk tensor store, instead of
        // 32 rows' scattered 32-byte stores; two buffers per warp, the older store must
        // have finished reading its buffer before the buffer is refilled
        uint8_t* ysb = ystage + (size_t(warp - 2) * 2 + ybuf) * 4096;
        if (p.tma_store) {
          if (lane == 0) bulk_wait_read<1>();
          __syncwarp();
        }
        for (int cb = cb0; cb < cb1; cb += 4) {
          const int ng = min(4, cb1 - cb);
          uint64_t mbits = 0;   // mask_direct: bit j of chunk i = (bf16 output > 0), 16 per chunk
          uint32_t r4[4][16];
#pragma unroll
          for (int i = 0; i < 4; ++i)
            if (i < ng) tmem_ld16_nowait(tbase + uint32_t(16 * (cb + i)), r4[i]);
#pragma unroll
          for (int i = 0; i < 4; ++i)
            if (i < ng) tmem_wait16(r4[i]);
          if (own || p.tma_store) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              if (i >= ng) break;
              const int c = 16 * (cb + i);
              float v[16];
#pragma unroll
              for (int j = 0; j < 16; j += 4) {
                const float4 bv = *reinterpret_cast<const float4*>(sbias + c + j);
                v[j] = __uint_as_float(r4[i][j]) + bv.x; v[j + 1] = __uint_as_float(r4[i][j + 1]) + bv.y;
                v[j + 2] = __uint_as_float(r4[i][j + 2]) + bv.z; v[j + 3] = __uint_as_float(r4[i][j + 3]) + bv.w;
              }
              if (p.relu) {
#pragma unroll
                for (int j = 0; j < 16; ++j) v[j] = fmaxf(v[j], 0.f);
              }
              if (p.row_div && own_deg > 0.f) {
#pragma unroll
                for (int j = 0; j < 16; ++j) v[j] = div_rn_rcp(v[j], own_deg, own_rdeg);
              }
              const int col = n0 + c;
              if (p.mask_direct) {   // the ReLU decision the backward reads: the stored bf16 value > 0
                uint32_t b16 = 0;
#pragma unroll
                for (int j = 0; j < 16; j += 2) {
                  const uint32_t w = pack_bf16x2(v[j], v[j + 1]);
                  b16 |= ((w & 0x7FFFu) && col + j < p.N ? 1u : 0u) << j;
                  b16 |= ((w & 0x7FFF0000u) && col + j + 1 < p.N ? 1u : 0u) << (j + 1);
                }
                mbits |= uint64_t(b16) << (16 * i);
              }
              if (p.tma_store) {   // rows past M: zeros (the box still covers them)
                const int u = 2 * (cb + i - cb0);
                uint8_t* rp = ysb + lane * 128;
                const bool ok = own != nullptr;
                *reinterpret_cast<uint4*>(rp + ((u ^ (lane & 7)) << 4)) =
                    ok ? make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                                    pack_bf16x2(v[6], v[7]))
                       : make_uint4(0, 0, 0, 0);
                *reinterpret_cast<uint4*>(rp + (((u + 1) ^ (lane & 7)) << 4)) =
                    ok ? make_uint4(pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]), pack_bf16x2(v[12], v[13]),
                                    pack_bf16x2(v[14], v[15]))
                       : make_uint4(0, 0, 0, 0);
              } else if (p.Yb) {
                uint16_t* d = reinterpret_cast<uint16_t*>(own) + col;
                if (col + 16 <= p.N && (reinterpret_cast<uintptr_t>(d) & 31) == 0) {
                  // the chunk's 32 bytes of this row as ONE sector-sized store (STG.256)
                  st_v8(d, pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                        pack_bf16x2(v[6], v[7]), pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]),
                        pack_bf16x2(v[12], v[13]), pack_bf16x2(v[14], v[15]));
                } else if (col + 16 <= p.N) {
                  reinterpret_cast<uint4*>(d)[0] = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
                                                              pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
                  reinterpret_cast<uint4*>(d)[1] = make_uint4(pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]),
                                                              pack_bf16x2(v[12], v[13]), pack_bf16x2(v[14], v[15]));
                } else {
#pragma unroll
                  for (int j = 0; j < 16; ++j)
                    if (col + j < p.N) d[j] = bf16_bits(v[j]);
                }
              } else {
                float* d = own + col;
                if (col + 16 <= p.N && (reinterpret_cast<uintptr_t>(d) & 31) == 0) {
#pragma unroll
                  for (int j = 0; j < 16; j += 8)
                    st_v8(d + j, __float_as_uint(v[j]), __float_as_uint(v[j + 1]), __float_as_uint(v[j + 2]),
                          __float_as_uint(v[j + 3]), __float_as_uint(v[j + 4]), __float_as_uint(v[j + 5]),
                          __float_as_uint(v[j + 6]), __float_as_uint(v[j + 7]));
                } else if (col + 16 <= p.N) {
#pragma unroll
                  for (int j = 0; j < 16; j += 4)
                    *reinterpret_cast<float4*>(d + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
                } else {
#pragma unroll
                  for (int j = 0; j < 16; ++j)
                    if (col + j < p.N) d[j] = v[j];
                }
              }
            }
          }
          if (p.mask_direct && own) {   // the group's <= 64 mask bits of this row: one 8-byte store
            uint16_t* mrow = p.mask + m_own * p.mask_pitch + (n0 + 16 * cb) / 16;
            if (ng == 4 && (reinterpret_cast<uintptr_t>(mrow) & 7) == 0) {
              *reinterpret_cast<uint2*>(mrow) = make_uint2(uint32_t(mbits), uint32_t(mbits >> 32));
            } else {
              for (int i = 0; i < ng; ++i) mrow[i] = uint16_t(mbits >> (16 * i));
            }
          }
        }
        fence_before();
        mbar_arrive(tempty + acc);
        if (++acc == p.nacc) { acc = 0; aph ^= 1; }
        if (p.tma_store) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // st.shared -> the TMA engine
          __syncwarp();
          if (lane == 0) {
            tma_store_2d(&mapY, ysb, n0 + 16 * cb0, int(t * BM + q * 32));
            bulk_commit();
          }
          ybuf ^= 1;
        }
        continue;
      }
      uint32_t r[16], rn[16];
      if (16 * h < p.BN) {
        tmem_ld16_nowait(tbase + uint32_t(16 * h), r);
        tmem_wait16(r);
      }
      for (int c = 16 * h; c < p.BN; c += 32) {
        const bool more = c + 32 < p.BN;
        if (more) tmem_ld16_nowait(tbase + uint32_t(c + 32), rn);
#pragma unroll
        for (int j = 0; j < 16; ++j) stg[lane * 17 + j] = __uint_as_float(r[j]);
        __syncwarp();
        const int col = n0 + c + cq;
        const float4 bv = *reinterpret_cast<const float4*>(sbias + c + cq);
#pragma unroll
        for (int it = 0; it < 4; ++it) {
          const int row = it * 8 + rsub;
          float* dst = reinterpret_cast<float*>(__shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(own), row));
          const float* sv = stg + row * 17 + cq;
          float4 v = make_float4(sv[0] + bv.x, sv[1] + bv.y, sv[2] + bv.z, sv[3] + bv.w);
          if (p.relu) { v.x = fmaxf(v.x, 0.f); v.y = fmaxf(v.y, 0.f); v.z = fmaxf(v.z, 0.f); v.w = fmaxf(v.w, 0.f); }
          if (p.row_div) {   // dZ / deg(v), the same correctly rounded quotient the pull formed per edge
            const float dg = __shfl_sync(0xffffffffu, own_deg, row), rd = __shfl_sync(0xffffffffu, own_rdeg, row);
            if (dg > 0.f) {
              v.x = div_rn_rcp(v.x, dg, rd); v.y = div_rn_rcp(v.y, dg, rd);
              v.z = div_rn_rcp(v.z, dg, rd); v.w = div_rn_rcp(v.w, dg, rd);
            }
          }
          if (p.mask) {   // 16 mask bits of (row, chunk) from the 4 lanes of the row segment
            uint32_t bits = (col < p.N && v.x > 0.f ? 1u : 0u) | (col + 1 < p.N && v.y > 0.f ? 2u : 0u) |
                            (col + 2 < p.N && v.z > 0.f ? 4u : 0u) | (col + 3 < p.N && v.w > 0.f ? 8u : 0u);
            bits <<= 4 * (lane & 3);
            bits |= __shfl_xor_sync(0xffffffffu, bits, 1);
            bits |= __shfl_xor_sync(0xffffffffu, bits, 2);
            if ((lane & 3) == 0 && dst && col < p.N) {
              const int64_t m = t * BM + q * 32 + row;
              p.mask[m * p.mask_pitch + (n0 + c) / 16] = uint16_t(bits);
            }
          }
          if (!dst || col >= p.N) continue;
          if (p.Yb) {
            uint16_t* db = reinterpret_cast<uint16_t*>(dst) + col;
            if (col + 4 <= p.N) {
              *reinterpret_cast<uint2*>(db) = make_uint2(pack_bf16x2(v.x, v.y), pack_bf16x2(v.z, v.w));
            } else {
              const float w4[4] = {v.x, v.y, v.z, v.w};
              for (int qq = 0; qq < 4 && col + qq < p.N; ++qq) {
                __nv_bfloat16 hh = __float2bfloat16_rn(w4[qq]);
                db[qq] = *reinterpret_cast<uint16_t*>(&hh);
              }
            }
            continue;
          }
          if (p.accumulate) {
            if (col + 4 <= p.N) {
              red_add_v4(dst + col, v.x, v.y, v.z, v.w);
            } else {
              atomicAdd(dst + col, v.x);
              if (col + 1 < p.N) atomicAdd(dst + col + 1, v.y);
              if (col + 2 < p.N) atomicAdd(dst + col + 2, v.z);
            }
          } else if (col + 4 <= p.N) {
            *reinterpret_cast<float4*>(dst + col) = v;
          } else {
            dst[col] = v.x;
            if (col + 1 < p.N) dst[col + 1] = v.y;
            if (col + 2 < p.N) dst[col + 2] = v.z;
          }
        }
        __syncwarp();
        if (more) {
          tmem_wait16(rn);
#pragma unroll
          for (int j = 0; j < 16; ++j) r[j] = rn[j];
        }
      }
      fence_before();
      mbar_arrive(tempty + acc);
      if (++acc == p.nacc) { acc = 0; aph ^= 1; }
    }
  }
  if (p.tma_store && warp >= 2 && lane == 0) bulk_wait_all();   // the output is written before the grid ends
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem_base, uint32_t(p.tmem_cols));
  }
}

// ------------------------------------------------------------ weight-gradient kernel
constexpr int WG_MAX_STAGES = 8;   // ring depth: as many stages as shared memory holds (runtime p.stages)

struct WgradParams {
  const int32_t* rows_dev;  // number of valid rows (device)
  int64_t rows_max;
  int d_out, d_in, BN, nbz, tmem_cols;
  int ones_col;             // Z column d_in holds 1.0: output column d_in is db
  uint32_t stage_bytes;     // A (2 x 8 KB) + B (nbz x 8 KB)
  int stages;               // ring depth (<= WG_MAX_STAGES)
  float* dW;                // [d_out x ldw] (accumulated)
  float* db;                // [d_out] (accumulated) or null
  int64_t ldw;
};

__global__ void __launch_bounds__(THREADS, 1)
    wgrad_kernel(const __grid_constant__ CUtensorMap mapG, const __grid_constant__ CUtensorMap mapZ, WgradParams p) {
  // PDL: barriers and TMEM are set up before griddepcontrol.wait (overlapping the
  // preceding kernel's tail); the row count and every operand are read after it
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);   // 1 KB aligned, still __shared__
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + size_t(p.stages) * p.stage_bytes);
  uint64_t* full = bars;
  uint64_t* empty = bars + WG_MAX_STAGES;
  uint64_t* tfull = bars + 2 * WG_MAX_STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tfull + 1);

  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int m0 = blockIdx.y * BM;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < p.stages; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapG)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapZ)) : "memory");
  }
  if (warp == 1) tmem_alloc(tmem_slot, uint32_t(p.tmem_cols));
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem_base = *tmem_slot;
  pdl_wait();
  pdl_launch();
  const int64_t rows = std::min<int64_t>(p.rows_max, int64_t(*p.rows_dev));
  const int64_t nkb_all = ceil_div(rows, BK);
  const int64_t per = ceil_div(nkb_all, int64_t(gridDim.x));
  const int64_t kb0 = int64_t(blockIdx.x) * per;
  const int64_t kb1 = std::min<int64_t>(nkb_all, kb0 + per);
  if (kb0 >= kb1) {   // uniform for the CTA: nothing to add
    __syncthreads();
    if (warp == 1) tmem_dealloc(tmem_base, uint32_t(p.tmem_cols));
    return;
  }

  if (warp == 0) {
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      // boxes entirely outside the matrices are not loaded: the MMA rows / columns
      // they feed are never read back by the epilogue
      const int na = (p.d_out - m0 > 64) ? 2 : 1;
      const int zcols = p.ones_col ? p.d_in + 1 : p.d_in;
      const int nz = int(ceil_div(zcols, 64));
      for (int64_t kb = kb0; kb < kb1; ++kb) {
        mbar_wait(empty + s, ph ^ 1);
        mbar_expect_tx(full + s, uint32_t(na + nz) * MNBLK);
        uint8_t* st = smem + size_t(s) * p.stage_bytes;
        const int y = int(kb * BK);
        for (int j = 0; j < na; ++j) tma_load_2d(st + j * MNBLK, &mapG, full + s, m0 + 64 * j, y);
        for (int j = 0; j < nz; ++j) tma_load_2d(st + 2 * MNBLK + j * MNBLK, &mapZ, full + s, j * 64, y);
        if (++s == p.stages) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    int s = 0;
    uint32_t ph = 0;
    for (int64_t kb = kb0; kb < kb1; ++kb) {
      mbar_wait(full + s, ph);
      fence_after();
      if (lane == 0) {
        const uint32_t a0 = smem_u32(smem + size_t(s) * p.stage_bytes);
        const uint32_t b0 = a0 + 2 * MNBLK;
#pragma unroll
        for (int kk = 0; kk < BK / 16; ++kk) {
          for (int n0 = 0; n0 < p.BN; n0 += 256) {
            const int nn = std::min(256, p.BN - n0);
            mma_bf16(tmem_base + uint32_t(n0), desc_mn(a0, kk), desc_mn(b0 + uint32_t(n0 / 64) * MNBLK, kk),
                     idesc_bf16(BM, nn, 1, 1), (kb > kb0 || kk) ? 1u : 0u);
          }
        }
        mma_commit(empty + s);
      }
      __syncwarp();
      if (++s == p.stages) { s = 0; ph ^= 1; }
    }
    if (lane == 0) mma_commit(tfull);
    __syncwarp();
  } else {
    // ---- epilogue: lane quarter q holds d_out rows m0 + 32q .. +31; 32-column
    // chunks staged in shared memory, then row-contiguous 16-B vector reductions
    const int q = warp & 3;
    float* stg = reinterpret_cast<float*>(tmem_slot + 4) + (warp - 2) * 32 * 33;
    const int rsub = lane >> 3, cq = (lane & 7) * 4;
    mbar_wait(tfull, 0);
    fence_after();
    const bool vec = (p.d_in & 3) == 0 && (p.ldw & 3) == 0 && (reinterpret_cast<uintptr_t>(p.dW) & 15) == 0;
    for (int c = 0; c < p.BN; c += 32) {
      uint32_t r[16];
      tmem_ld16(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(c), r);
#pragma unroll
      for (int j = 0; j < 16; ++j) stg[lane * 33 + j] = __uint_as_float(r[j]);
      if (c + 16 < p.BN) {
        tmem_ld16(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(c + 16), r);
#pragma unroll
        for (int j = 0; j < 16; ++j) stg[lane * 33 + 16 + j] = __uint_as_float(r[j]);
      }
      __syncwarp();
      const int col = c + cq;
#pragma unroll
      for (int it = 0; it < 8; ++it) {
        const int row = it * 4 + rsub;
        const int o = m0 + q * 32 + row;
        if (o >= p.d_out || col > p.d_in) continue;
        const float* sv = stg + row * 33 + cq;
        float* w = p.dW + int64_t(o) * p.ldw + col;
        if (vec && col + 4 <= p.d_in) {
          red_add_v4(w, sv[0], sv[1], sv[2], sv[3]);
        } else {
          for (int j = 0; j < 4; ++j) {
            if (col + j < p.d_in) atomicAdd(w + j, sv[j]);
            else if (col + j == p.d_in && p.ones_col && p.db) atomicAdd(p.db + o, sv[j]);
          }
        }
      }
      __syncwarp();
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem_base, uint32_t(p.tmem_cols));
  }
}

}  // namespace tc

int tc_gemm_supported(int N, int K) { return N >= 1 && N <= 256 && K >= 1 && K <= 256; }

cudaError_t launch_tc_gemm(const TcGemmArgs& a, cudaStream_t st) {
  using namespace tc;
  if (!tc_gemm_supported(a.N, a.K)) return cudaErrorInvalidValue;
  if ((a.z_pitch * 2) % 16 || (a.w_pitch * 2) % 16 || (a.y_pitch * 4) % 16) return cudaErrorInvalidValue;
  if (a.Yb && ((a.yb_pitch * 2) % 8 || a.out_rank || a.accumulate)) return cudaErrorInvalidValue;
  const int BN_all = int(round_up(a.N, 16));
  const int nkb = int(ceil_div(a.K, BK));
  // few M tiles (small blocks, a requester's own rows): split the columns over CTAs so
  // that more SMs share the tile's epilogue; slices stay multiples of 64 columns
  const int64_t tiles = std::max<int64_t>(1, ceil_div(a.M_max, BM));
  int n_split = 1;
  while (n_split < 4 && tiles * n_split * 2 <= sm_count() && BN_all % (64 * n_split * 2) == 0) n_split *= 2;
  // 128-column slices even with many tiles: A/B on the products step (APT_PROJ_SPLIT =
  // 1 / 2 / 4 for every projection and dZ): 0.230 / 0.221 / 0.229 ms
  static const int force_split = [] { const char* v = std::getenv("APT_PROJ_SPLIT"); return v ? atoi(v) : -1; }();
  const int want_split = force_split >= 0 ? force_split : 2;
  if (want_split > n_split && BN_all % (64 * want_split) == 0) n_split = want_split;
  const int BN = BN_all / n_split;
  static const int epi_staged = [] { const char* v = std::getenv("APT_EPI_STAGED"); return v ? atoi(v) : 0; }();
  CUtensorMap ma, mb;
  if (!make_map(&ma, a.Z, a.K, std::max<int64_t>(a.M_max, 1), a.z_pitch, BK, BM)) return cudaErrorInvalidValue;
  uint32_t b_kb_bytes;
  if (a.w_mn) {
    // W stored [K x N] (N contiguous): boxes of 64 N x 64 K
    if (!make_map(&mb, a.W, a.N, a.K, a.w_pitch, 64, BK)) return cudaErrorInvalidValue;
    b_kb_bytes = uint32_t(ceil_div(BN, 64)) * MNBLK;
  } else {
    if (!make_map(&mb, a.W, a.K, a.N, a.w_pitch, BK, BN)) return cudaErrorInvalidValue;
    b_kb_bytes = uint32_t(BN) * 128;
  }
  // two CTAs per SM when they fit (2-stage ring, one TMEM accumulator each): one CTA's
  // loads and MMAs overlap the other's epilogue
  static const int two_cta = [] { const char* v = std::getenv("APT_PROJ_2CTA"); return v ? atoi(v) : 0; }();   // off: measured slower end to end (the overlapped sampling then lands on the backward)
  // bf16 rows in 128-column slices leave through TMA stores (APT_EPI_TMA=0: per-row 32-byte
  // stores, A/B)
  static const int epi_tma = [] { const char* v = std::getenv("APT_EPI_TMA"); return v ? atoi(v) : 1; }();
  CUtensorMap my;
  int tma_store = 0;
  // ReLU bits of bf16 rows from the direct epilogue (8-byte stores of 64 bits per row and warp)
  const int mask_direct = (a.mask && a.Yb && !a.out_rank && !a.accumulate && !epi_staged && BN % 64 == 0 &&
                           (a.mask_pitch % 4) == 0) ? 1 : 0;
  if (epi_tma && a.Yb && BN == 128 && !a.out_rank && !a.accumulate && (!a.mask || mask_direct) && !epi_staged &&
      (a.yb_pitch * 2) % 16 == 0 && (reinterpret_cast<uintptr_t>(a.Yb) & 15) == 0 &&
      make_map(&my, a.Yb, a.N, std::max<int64_t>(a.M_max, 1), a.yb_pitch, 64, 32))
    tma_store = 1;
  else
    my = ma;   // unused
  auto smem_of = [&](int st) {
    return 1024 + size_t(st) * A_STAGE_BYTES + size_t(nkb) * b_kb_bytes + 128 + 1024 + 8 * 32 * 17 * 4 +
           (tma_store ? 1024 + 8 * 2 * 4096 : 0);
  };
  int stages = STAGES, nacc = 2, per_sm = 1;
  if (two_cta && !a.w_mn && smem_of(2) <= 113 * 1024 && BN <= 256 && tiles * n_split > sm_count()) {
    stages = 2;
    nacc = 1;
    per_sm = 2;
  }
  int cols = 32;
  while (cols < nacc * BN) cols <<= 1;
  RowParams p{a.M_max, a.M_dev, a.N, BN, nkb, cols, a.w_mn, stages, nacc, b_kb_bytes, a.bias, a.relu, a.Y, a.y_pitch,
              a.out_base, a.out_rank, a.out_row, a.accumulate, n_split, a.mask, a.mask_pitch, mask_direct,
              a.row_div_indptr,
              a.Yb, a.yb_pitch, a.b_early, epi_staged, tma_store};
  const size_t smem = smem_of(stages);   // + epilogue staging
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(rowtile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set = true;
  }
  const int grid = int(std::min<int64_t>(tiles * n_split, ((per_sm * sm_count()) / n_split) * n_split));
  launch_pdl(rowtile_kernel, dim3(grid), dim3(ROW_THREADS), smem, st, ma, mb, my, p);
  return cudaGetLastError();
}

int tc_wgrad_supported(int d_out, int d_in) { return d_out >= 1 && d_out <= 256 && d_in >= 1 && d_in + 1 <= 320; }

cudaError_t launch_tc_wgrad(const TcWgradArgs& a, cudaStream_t st) {
  using namespace tc;
  if (!tc_wgrad_supported(a.d_out, a.d_in)) return cudaErrorInvalidValue;
  if ((a.g_pitch * 2) % 16 || (a.z_pitch * 2) % 16) return cudaErrorInvalidValue;
  const int zcols = a.db ? a.d_in + 1 : a.d_in;     // column d_in of Z is all ones (db)
  if (a.db && a.z_pitch < zcols) return cudaErrorInvalidValue;
  const int BN = int(round_up(zcols, 16));
  const int nbz = int(ceil_div(BN, 64));
  int cols = 32;
  while (cols < BN) cols <<= 1;
  CUtensorMap mg, mz;
  const int64_t rows = std::max<int64_t>(a.rows_max, 1);
  if (!make_map(&mg, a.G, a.d_out, rows, a.g_pitch, 64, BK)) return cudaErrorInvalidValue;
  if (!make_map(&mz, a.Z, zcols, rows, a.z_pitch, 64, BK)) return cudaErrorInvalidValue;
  const uint32_t stage = uint32_t(2 + nbz) * MNBLK;
  WgradParams p{a.rows_dev, a.rows_max, a.d_out, a.d_in, BN, nbz, cols, a.db ? 1 : 0, stage, 0, a.dW, a.db,
                a.ldw > 0 ? a.ldw : a.d_in};
  // ring depth: as many stages as fit (more bytes in flight per SM: the loads are the
  // latency of this kernel), A/B via APT_WG_STAGES
  static const int want = [] { const char* v = std::getenv("APT_WG_STAGES"); return v ? atoi(v) : 3; }();   // 3 / 8: 0.2199 / 0.2205 ms
  const size_t fixed = 1024 + size_t(2 * WG_MAX_STAGES + 1) * 8 + 16 + 4 * 32 * 33 * 4;
  int stages = std::max(2, std::min<int>(want, int((227 * 1024 - fixed) / stage)));
  stages = std::min(stages, WG_MAX_STAGES);
  p.stages = stages;
  const size_t smem = fixed + size_t(stages) * stage;
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(wgrad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set = true;
  }
  const int mt = int(ceil_div(a.d_out, BM));
  const int64_t kbs = std::max<int64_t>(1, ceil_div(a.rows_max, BK));
  // row splits: one CTA per SM (A/B APT_WG_SPLITS_PER_SM = 1 / 2: 0.207 / 0.224 ms; ring depth 3 / 6: same)
  static const int per_sm = [] { const char* v = std::getenv("APT_WG_SPLITS_PER_SM"); return v ? std::max(1, atoi(v)) : 1; }();
  // at least APT_WG_MIN_KB k-blocks per split: a small block (the upper layers' few thousand
  // rows) over every SM leaves each CTA ~1 k-block and every dW element ~74 contended
  // reductions; fewer, longer splits pipeline their loads and reduce less
  // (A/B on the products step, 2 x 2 runs: 1 / 4 / 8 / 16 -> 0.1638 / 0.1630 / 0.1642 / 0.1663 ms)
  static const int min_kb = [] { const char* v = std::getenv("APT_WG_MIN_KB"); return v ? std::max(1, atoi(v)) : 4; }();
  const int splits = int(std::max<int64_t>(
      1, std::min<int64_t>(ceil_div(kbs, int64_t(min_kb)), int64_t(per_sm) * sm_count() / mt)));
  launch_pdl(wgrad_kernel, dim3(dim3(splits, mt)), dim3(THREADS), smem, st, mg, mz, p);
  return cudaGetLastError();
}

}  // namespace apt
