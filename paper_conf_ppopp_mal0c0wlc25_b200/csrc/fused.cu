// fused.cu -- the first layer's forward as ONE kernel (S6+S7+S8): feature gather,
// GraphSAGE mean, tcgen05 projection, bias + ReLU epilogue.
//
//   h1[v] = ReLU( W * mean_{u in N_s(v)} x[u] + b )        (Eq. 1)
//
// Persistent CTAs (one per SM), 128-destination tiles, warp-specialised:
//  * warps 5..28 (gatherers, 48 lane groups of 16): the mean of one destination
//    row per group at a time, straight from HBM with 16-B vector loads (one edge
//    pointer per lane, broadcast by shuffles, 4 loads in flight per lane -- the
//    agg_kernel scheme); fp32 sums, IEEE RN division by the sampled degree (O5),
//    bf16 rounding; the row goes to global Z (kept for the weight gradient, with its
//    all-ones bias column) and into the tile's UMMA A operand in shared memory
//    (K-major, 128-B swizzle), double-buffered per tile.
//    (TMA tile::gather4 was measured first: for 208-B rows it peaks near 2.5 TB/s
//    per device, 4x below what the load/store units reach on the same gather.)
//  * warp 0: W to shared memory once (TMA), TMEM allocation and the single-thread
//    tcgen05.mma issue (M=128, N<=256, K=16 slices) into a double-buffered TMEM
//    accumulator.
//  * warps 1..4 (epilogue): tcgen05.ld -> +bias -> ReLU -> fp32 h1, staged in
//    shared memory for row-contiguous stores.
// Z never makes the round trip through HBM between the mean and the projection,
// and the gather of tile i+1 overlaps the MMA and epilogue of tile i.
// Applies to a single-shard bf16 store with rows of <= 128 features (products,
// papers d=64); other cases use agg_kernel + rowtile_kernel.
#include "common.cuh"
#include "kernels.h"
#include "tc_common.cuh"

namespace apt {
namespace tc {

constexpr int FU_GW = 24;                    // gatherer warps (48 groups of 16 lanes)
constexpr int FU_EPI_WARPS = 4;
constexpr int FU_THREADS = (1 + FU_EPI_WARPS + FU_GW) * 32;
constexpr int FU_GROUPS = FU_GW * 2;

struct FusedParams {
  const int32_t* cnt; const int32_t* nbr; int k;
  const int32_t* n_dev; int64_t M_max;
  const uint8_t* feat; int64_t row_bytes;      // bf16 store, single shard
  int d, V, nkb, nks;
  int N, BN; uint32_t w_kb_bytes; int tmem_cols;
  const float* bias; int relu;
  float* Y; int64_t y_pitch;
  uint16_t* Z; int64_t z_pitch; int z_ones;
};

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void sts_v4(void* p, uint4 v) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(smem_u32(p)), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

__global__ void __launch_bounds__(FU_THREADS, 1)
    sage_l1_kernel(const __grid_constant__ CUtensorMap mapW, FusedParams p) {
  APT_PDL_PROLOGUE();
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t a_stage = uint32_t(p.nkb) * 16384u;
  uint8_t* sA = smem;                                            // 2 A stages
  uint8_t* sW = sA + 2 * a_stage;                                // resident W
  float* stg_all = reinterpret_cast<float*>(sW + uint32_t(p.nkb) * p.w_kb_bytes);
  uint64_t* bars = reinterpret_cast<uint64_t*>(stg_all + FU_EPI_WARPS * 32 * 17);
  uint64_t* wfull = bars;
  uint64_t* afull = bars + 1;     // [2]
  uint64_t* aempty = bars + 3;    // [2]
  uint64_t* tfull = bars + 5;     // [2]
  uint64_t* tempty = bars + 7;    // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 9);

  const int warp = threadIdx.x >> 5, lane = lane_id();
  const int64_t M = std::min<int64_t>(p.M_max, int64_t(*p.n_dev));
  const int64_t ntiles = ceil_div(M, BM);

  if (warp == 0) {
    if (lane == 0) {
      mbar_init(wfull, 1);
      for (int i = 0; i < 2; ++i) {
        mbar_init(afull + i, FU_GW);
        mbar_init(aempty + i, 1);
        mbar_init(tfull + i, 1);
        mbar_init(tempty + i, FU_EPI_WARPS * 32);
      }
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapW)) : "memory");
    }
    __syncwarp();
    tmem_alloc(tmem_slot, uint32_t(p.tmem_cols));
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ---------------------------------------------------------------- W + MMA issuer
    if (ntiles > int64_t(blockIdx.x)) {
      if (lane == 0) {
        mbar_expect_tx(wfull, uint32_t(p.nkb) * p.w_kb_bytes);
        for (int kb = 0; kb < p.nkb; ++kb) tma_load_2d(sW + kb * p.w_kb_bytes, &mapW, wfull, kb * BK, 0);
      }
      const uint32_t idesc = idesc_bf16(BM, p.BN, 0, 0);
      mbar_wait(wfull, 0);
      fence_after();
      uint32_t it = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
        const int s = it & 1, acc = it & 1;
        const uint32_t ph = (it >> 1) & 1;
        mbar_wait(tempty + acc, ph ^ 1);
        mbar_wait(afull + s, ph);
        fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(sA + s * a_stage), b0 = smem_u32(sW);
          const uint32_t d = tmem_base + uint32_t(acc * p.BN);
          for (int ks = 0; ks < p.nks; ++ks) {
            const int kb = ks >> 2, kk = ks & 3;
            mma_bf16(d, desc_k(a0 + kb * 16384, kk), desc_k(b0 + kb * p.w_kb_bytes, kk), idesc, ks > 0);
          }
          mma_commit(aempty + s);
          mma_commit(tfull + acc);
        }
        __syncwarp();
      }
    }
  } else if (warp <= FU_EPI_WARPS) {
    // ---------------------------------------------------------------- epilogue (warps 1..4)
    const int q = warp & 3;
    float* stg = stg_all + (warp - 1) * 32 * 17;
    const int rsub = lane >> 2, cq = (lane & 3) * 4;
    uint32_t it = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int acc = it & 1;
      mbar_wait(tfull + acc, (it >> 1) & 1);
      fence_after();
      const int64_t m_own = t * BM + q * 32 + lane;
      float* own = m_own < M ? p.Y + m_own * p.y_pitch : nullptr;
      for (int c = 0; c < p.BN; c += 16) {
        uint32_t rr[16];
        tmem_ld16(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * p.BN + c), rr);
#pragma unroll
        for (int jj = 0; jj < 16; ++jj) stg[lane * 17 + jj] = __uint_as_float(rr[jj]);
        __syncwarp();
        const int col = c + cq;
        float4 bv = make_float4(0.f, 0.f, 0.f, 0.f);
        if (p.bias) {
          if (col + 4 <= p.N) bv = *reinterpret_cast<const float4*>(p.bias + col);
          else {
            if (col < p.N) bv.x = p.bias[col];
            if (col + 1 < p.N) bv.y = p.bias[col + 1];
            if (col + 2 < p.N) bv.z = p.bias[col + 2];
          }
        }
#pragma unroll
        for (int k4 = 0; k4 < 4; ++k4) {
          const int row = k4 * 8 + rsub;
          float* dst = reinterpret_cast<float*>(__shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(own), row));
          if (!dst || col >= p.N) continue;
          const float* sv = stg + row * 17 + cq;
          float4 v = make_float4(sv[0] + bv.x, sv[1] + bv.y, sv[2] + bv.z, sv[3] + bv.w);
          if (p.relu) { v.x = fmaxf(v.x, 0.f); v.y = fmaxf(v.y, 0.f); v.z = fmaxf(v.z, 0.f); v.w = fmaxf(v.w, 0.f); }
          if (col + 4 <= p.N) {
            *reinterpret_cast<float4*>(dst + col) = v;
          } else {
            dst[col] = v.x;
            if (col + 1 < p.N) dst[col + 1] = v.y;
            if (col + 2 < p.N) dst[col + 2] = v.z;
          }
        }
        __syncwarp();
      }
      fence_before();
      mbar_arrive(tempty + acc);
    }
  } else {
    // ---------------------------------------------------------------- gatherers (warps 5..)
    const int grp = (warp - 1 - FU_EPI_WARPS) * 2 + (lane >> 4), sub = lane >> 4, l = lane & 15;
    uint32_t it = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int s = it & 1;
      mbar_wait(aempty + s, ((it >> 1) & 1) ^ 1);   // the MMA of tile it-2 has consumed this stage
      uint8_t* A = sA + s * a_stage;
      // rows grp, grp + 48, ... of the tile; both half-warps run the same trip count
      for (int r0 = 0; r0 < BM; r0 += FU_GROUPS) {
        const int r = r0 + grp;
        const int64_t i = t * BM + r;
        const bool valid = r < BM && i < M;
        const int cnt = valid ? p.cnt[i] : 0;
        int cmax = cnt;
        cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, 16));
        float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
        for (int e0 = 0; e0 < cmax; e0 += 16) {
          const char* rp = nullptr;
          if (valid && e0 + l < cnt) rp = reinterpret_cast<const char*>(p.feat) + int64_t(p.nbr[i * p.k + e0 + l]) * p.row_bytes;
          const int m = min(16, cmax - e0);
          for (int j = 0; j < m; j += 4) {
            uint4 v[4];
#pragma unroll
            for (int q4 = 0; q4 < 4; ++q4) {
              const char* rr = reinterpret_cast<const char*>(
                  __shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(rp), sub * 16 + ((j + q4) & 15)));
              v[q4] = (j + q4 < m && rr != nullptr && l < p.V) ? ld_nc_v4(rr + l * 16) : make_uint4(0, 0, 0, 0);
            }
#pragma unroll
            for (int q4 = 0; q4 < 4; ++q4) {
              acc[0] += bf16_lo(v[q4].x); acc[1] += bf16_hi(v[q4].x);
              acc[2] += bf16_lo(v[q4].y); acc[3] += bf16_hi(v[q4].y);
              acc[4] += bf16_lo(v[q4].z); acc[5] += bf16_hi(v[q4].z);
              acc[6] += bf16_lo(v[q4].w); acc[7] += bf16_hi(v[q4].w);
            }
          }
        }
        if (r >= BM) continue;
        uint4 zb = make_uint4(0, 0, 0, 0);
        if (valid && l < p.V && cnt > 0) {
          const float fdeg = float(cnt), rdeg = __frcp_rn(fdeg);
          float z[8];
#pragma unroll
          for (int q = 0; q < 8; ++q) z[q] = div_rn_rcp(acc[q], fdeg, rdeg);
          zb = make_uint4(pack_bf16x2(z[0], z[1]), pack_bf16x2(z[2], z[3]), pack_bf16x2(z[4], z[5]),
                          pack_bf16x2(z[6], z[7]));
        }
        if (valid && l < p.V) {
          uint16_t* zr = p.Z + i * p.z_pitch;
          if (l * 8 + 8 <= p.d) {
            *reinterpret_cast<uint4*>(zr + l * 8) = zb;
          } else {
            const uint32_t w[4] = {zb.x, zb.y, zb.z, zb.w};
            for (int q = 0; q < 8 && l * 8 + q < p.d; ++q) zr[l * 8 + q] = uint16_t(w[q >> 1] >> ((q & 1) * 16));
          }
          if (p.z_ones && l == 0) zr[p.d] = 0x3F80;   // bf16 1.0: bias-gradient column
        }
        // the tile's UMMA A operand: 16-B chunk l of row r, K-major SW128 layout
        if (l < 8 * p.nkb) {
          uint8_t* dst = A + (l >> 3) * 16384 + (r >> 3) * 1024 + (r & 7) * 128 + (((l & 7) ^ (r & 7)) << 4);
          sts_v4(dst, l < p.V ? zb : make_uint4(0, 0, 0, 0));
        }
      }
      fence_proxy_async();                          // generic-proxy smem writes -> tensor-core (async) proxy
      __syncwarp();
      if (lane == 0) mbar_arrive(afull + s);
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 0) {
    fence_after();
    tmem_dealloc(tmem_base, uint32_t(p.tmem_cols));
  }
}

}  // namespace tc

cudaError_t launch_sage_l1(const FusedL1Args& a, cudaStream_t st) {
  using namespace tc;
  const int V = int(ceil_div(a.d, 8));
  if (a.d < 1 || V > 16 || a.N < 1 || a.N > 256 || a.k < 1 || a.row_elems < a.d || (a.row_elems % 8) ||
      (a.z_pitch % 8) || (a.y_pitch % 4) || (a.w_pitch % 8))
    return cudaErrorNotSupported;
  const int BN = int(round_up(a.N, 16));
  const int nks = int(ceil_div(a.d, 16));
  const int nkb = int(ceil_div(nks * 16, 64));
  const uint32_t w_kb = uint32_t(BN) * 128;
  const size_t smem = 1024 + size_t(2) * nkb * 16384 + size_t(nkb) * w_kb + FU_EPI_WARPS * 32 * 17 * 4 + 16 * 8;
  if (smem > 227 * 1024) return cudaErrorNotSupported;
  int cols = 32;
  while (cols < 2 * BN) cols <<= 1;
  CUtensorMap mw;
  if (!make_map(&mw, a.Wb, a.d, a.N, a.w_pitch, BK, BN)) return cudaErrorNotSupported;
  FusedParams p{a.cnt, a.nbr, a.k, a.n_dev, a.M_max, reinterpret_cast<const uint8_t*>(a.feat),
                int64_t(a.row_elems) * 2, a.d, V, nkb, nks, a.N, BN, w_kb, cols, a.bias, a.relu, a.Y, a.y_pitch,
                a.Z, a.z_pitch, a.z_ones};
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(sage_l1_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr = true;
  }
  const int64_t tiles = std::max<int64_t>(1, ceil_div(a.M_max, BM));
  const int grid = int(std::min<int64_t>(tiles, sm_count()));
  launch_pdl(sage_l1_kernel, dim3(grid), dim3(FU_THREADS), smem, st, mw, p);
  return cudaGetLastError();
}

}  // namespace apt
