// Persistent, warp-specialised tcgen05 HGEMM for sm_100a.
//
// Kernel coordinates.  The kernel computes a ROW-MAJOR tile matrix
//     D[M x N] = alpha * Ak[M x K] * Bk[N x K]^T + beta * D,      D[r][c] at D + r*ldd + c
// where Ak feeds the UMMA "A" operand (rows -> TMEM lanes) and Bk the UMMA
// "B" operand (rows -> TMEM columns).  The host maps the column-major ABI
// C = op(A) op(B) onto it as D = C^T (M = n, N = m, ldd = ldc, Ak = op(B)^T,
// Bk = op(A)), so each epilogue thread owns one output column of C and
// writes contiguous runs of m.
//
// Paper mapping:
//   Alg. 1 P:248-272 two-level blocking      -> CTA tile 128 x BN (x2 for the CTA pair),
//                                               k-block BK = 64 (one 128-B swizzle atom)
//   SVI-A.2 P:274 grid of ceil(m/bm) x ceil(n/bn) blocks
//                                             -> persistent clusters walking an
//                                               L2-grouped raster (future work at P:460)
//   SVI-B P:361-363 prefetching              -> STAGES-deep TMA ring with full/empty mbarriers
//   SVI-C P:367-379 CPI-based interleaving   -> warp specialisation (TMA warp, MMA warp,
//                                               4 epilogue warps); no issue-slot scheduling left
//   SVI-D P:381-397 padded smem layout       -> TMA SWIZZLE_128B + UMMA SW128 descriptors
//   SIV Eq. 2 P:104 HMMA.1688               -> tcgen05.mma.kind::f16, FP32 accumulation in TMEM
//
// Warp roles (192 threads, 1 CTA per SM):
//   warp 0     : TMA producer (one elected lane)
//   warp 1     : TMEM allocator; in the leader CTA, the MMA issuer (one lane)
//   warps 2..5 : epilogue, TMEM lanes 32*(warp%4) .. +31
// Pipelines: smem ring full[s]/empty[s]; accumulator double buffer
// tmem_full[2]/tmem_empty[2] so the epilogue of tile i overlaps the
// mainloop of tile i+1.
#pragma once
#include <cuda_fp16.h>

#include "ptx.cuh"

namespace hg {

struct TcParams {
  int32_t M, N, K;                 // D is M x N, reduction length K
  int32_t num_m_tiles, num_n_tiles;  // in cluster tiles (128*CG x BN)
  int32_t num_k_blocks;
  int32_t group_m;                 // raster group height, in m-tiles
  float alpha, beta;
  void *D;
  int64_t ldd;
};

// UMMA shared-memory descriptor, SWIZZLE_128B, K-major operand.
// Rows of 128 B (64 FP16 along K); 8-row core groups 1024 B apart (SBO).
// LBO is unused for a swizzled K-major operand whose K extent per MMA
// (16 FP16 = 32 B) lies inside one swizzle atom.
__device__ __forceinline__ uint64_t sdesc_k_sw128(uint32_t saddr) {
  uint64_t d = 0;
  d |= static_cast<uint64_t>((saddr >> 4) & 0x3FFFu);
  d |= static_cast<uint64_t>(1u) << 16;              // LBO = 16 B (ignored)
  d |= static_cast<uint64_t>(1024u >> 4) << 32;      // SBO = 1024 B
  d |= static_cast<uint64_t>(1u) << 46;              // descriptor version 1 (sm_100)
  d |= static_cast<uint64_t>(2u) << 61;              // layout: SWIZZLE_128B
  return d;
}
// UMMA shared-memory descriptor, SWIZZLE_128B, MN-major operand.
// Each TMA box is 64 K-rows x 128 B (64 FP16 along M/N); 8 K-rows form a
// 1024-B swizzle atom (SBO); consecutive 64-wide M/N blocks are `lbo` bytes apart.
__device__ __forceinline__ uint64_t sdesc_mn_sw128(uint32_t saddr, uint32_t lbo) {
  uint64_t d = 0;
  d |= static_cast<uint64_t>((saddr >> 4) & 0x3FFFu);
  d |= static_cast<uint64_t>((lbo >> 4) & 0x3FFFu) << 16;
  d |= static_cast<uint64_t>(1024u >> 4) << 32;
  d |= static_cast<uint64_t>(1u) << 46;
  d |= static_cast<uint64_t>(2u) << 61;
  return d;
}

// Instruction descriptor for kind::f16: D FP32, A/B FP16, majorness, N, M.
template <int M, int N, bool A_MN, bool B_MN>
__host__ __device__ constexpr uint32_t make_idesc_f16() {
  return (1u << 4)                                  // c_format = F32
         | (0u << 7) | (0u << 10)                   // a_format = b_format = F16
         | ((A_MN ? 1u : 0u) << 15) | ((B_MN ? 1u : 0u) << 16)
         | (static_cast<uint32_t>(N >> 3) << 17)    // N >> 3
         | (static_cast<uint32_t>(M >> 4) << 24);   // M >> 4
}

__device__ __forceinline__ void tile_coords(int t, const TcParams &p, int &tm, int &tn) {
  const int per_group = p.group_m * p.num_n_tiles;
  const int g = t / per_group;
  const int first_m = g * p.group_m;
  const int gsz = min(p.num_m_tiles - first_m, p.group_m);
  const int r = t - g * per_group;
  tm = first_m + r % gsz;
  tn = r / gsz;
}

__device__ __forceinline__ uint32_t pack_half2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);  // cvt.rn.f16x2.f32: RN-even, overflow -> inf
  return *reinterpret_cast<uint32_t *>(&h);
}

// Epilogue for one thread: 32 consecutive columns [col, col+32) of row `row`.
template <bool OUT_F32>
__device__ __forceinline__ void store_chunk(const TcParams &p, int row, int col, const uint32_t (&v)[32]) {
  if (row >= p.M || col >= p.N) return;
  const int ncol = min(32, p.N - col);
  const float alpha = p.alpha, beta = p.beta;
  if constexpr (OUT_F32) {
    float *dst = static_cast<float *>(p.D) + static_cast<int64_t>(row) * p.ldd + col;
    if (ncol == 32) {
      float4 *d4 = reinterpret_cast<float4 *>(dst);
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        float4 o;
        o.x = alpha * __uint_as_float(v[4 * q + 0]);
        o.y = alpha * __uint_as_float(v[4 * q + 1]);
        o.z = alpha * __uint_as_float(v[4 * q + 2]);
        o.w = alpha * __uint_as_float(v[4 * q + 3]);
        if (beta != 0.0f) {
          const float4 c = d4[q];
          o.x = fmaf(beta, c.x, o.x);
          o.y = fmaf(beta, c.y, o.y);
          o.z = fmaf(beta, c.z, o.z);
          o.w = fmaf(beta, c.w, o.w);
        }
        d4[q] = o;
      }
    } else {
#pragma unroll
      for (int j = 0; j < 32; ++j) {
        if (j < ncol) {
          float o = alpha * __uint_as_float(v[j]);
          if (beta != 0.0f) o = fmaf(beta, dst[j], o);
          dst[j] = o;
        }
      }
    }
  } else {
    __half *dst = static_cast<__half *>(p.D) + static_cast<int64_t>(row) * p.ldd + col;
    if (ncol == 32) {
      uint4 *d4 = reinterpret_cast<uint4 *>(dst);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        float f[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) f[e] = alpha * __uint_as_float(v[8 * q + e]);
        if (beta != 0.0f) {
          const uint4 c = d4[q];
          const __half2 *ch = reinterpret_cast<const __half2 *>(&c);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 cf = __half22float2(ch[e]);
            f[2 * e] = fmaf(beta, cf.x, f[2 * e]);
            f[2 * e + 1] = fmaf(beta, cf.y, f[2 * e + 1]);
          }
        }
        uint4 o;
        o.x = pack_half2(f[0], f[1]);
        o.y = pack_half2(f[2], f[3]);
        o.z = pack_half2(f[4], f[5]);
        o.w = pack_half2(f[6], f[7]);
        d4[q] = o;
      }
    } else {
#pragma unroll
      for (int j = 0; j < 32; ++j) {
        if (j < ncol) {
          float o = alpha * __uint_as_float(v[j]);
          if (beta != 0.0f) o = fmaf(beta, __half2float(dst[j]), o);
          dst[j] = __float2half_rn(o);
        }
      }
    }
  }
}

template <int BN, int CG>
struct TcShape {
  static constexpr int BM = 128;  // rows per CTA (TMEM lanes)
  static constexpr int BK = 64;   // FP16 per 128-B swizzle atom
  static constexpr int BN_CTA = BN / CG;
  static constexpr uint32_t A_BYTES = BM * BK * 2;
  static constexpr uint32_t B_BYTES = BN_CTA * BK * 2;
  static constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (STAGE_BYTES <= 32768) ? 6 : 4;
  static constexpr uint32_t TMEM_COLS = (2 * BN <= 64) ? 64 : (2 * BN <= 128) ? 128 : (2 * BN <= 256) ? 256 : 512;
  static constexpr uint32_t SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*barriers*/ + 1024 /*alignment*/;
  static_assert(BN % 32 == 0 && BN >= 64 && BN <= 256, "BN");
  static_assert(BN_CTA % 64 == 0, "BN_CTA");
};

template <int BN, int CG, bool A_MN, bool B_MN, bool OUT_F32>
__global__ void __launch_bounds__(192, 1)
    hgemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    const TcParams p) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  using S = TcShape<BN, CG>;
  constexpr int BM = S::BM;
  constexpr int BK = S::BK;
  constexpr int BN_CTA = S::BN_CTA;
  constexpr int STAGES = S::STAGES;
  constexpr uint32_t A_BYTES = S::A_BYTES;
  constexpr uint32_t STAGE_BYTES = S::STAGE_BYTES;
  constexpr uint32_t IDESC = make_idesc_f16<BM * CG, BN, A_MN, B_MN>();
  // Per-K=16 advance of the descriptor start address (in bytes).
  constexpr uint32_t A_KSTEP = A_MN ? 16 * 128 : 32;
  constexpr uint32_t B_KSTEP = B_MN ? 16 * 128 : 32;

  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw_u32 = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw_u32 & 1023u)) & 1023u);
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + STAGES * STAGE_BYTES);
  uint64_t *empty = full + STAGES;
  uint64_t *tfull = empty + STAGES;
  uint64_t *tempty = tfull + 2;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tempty + 2);

  const uint32_t warp = warp_id();
  const uint32_t lane = lane_id();
  const uint32_t rank = (CG == 2) ? cluster_ctarank() : 0u;
  const int cluster_id = static_cast<int>(blockIdx.x) / CG;
  const int num_clusters = static_cast<int>(gridDim.x) / CG;
  const int num_tiles = p.num_m_tiles * p.num_n_tiles;

  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
  }
  if (warp == 1) {
    if (lane == 0) {
      for (int s = 0; s < STAGES; ++s) {
        mbar_init(&full[s], 1);
        mbar_init(&empty[s], 1);
      }
      for (int a = 0; a < 2; ++a) {
        mbar_init(&tfull[a], 1);
        mbar_init(&tempty[a], 4 * CG);
      }
      fence_mbarrier_init();
    }
    __syncwarp();
    tmem_alloc<CG>(smem_u32(tmem_slot), S::TMEM_COLS);
  }
  tc_fence_before();
  if constexpr (CG == 2) cluster_sync(); else __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      const uint64_t pol = l2_policy_evict_normal();
      uint32_t stage = 0, phase = 0;
      for (int t = cluster_id; t < num_tiles; t += num_clusters) {
        int tm, tn;
        tile_coords(t, p, tm, tn);
        const int a_row = tm * BM * CG + static_cast<int>(rank) * BM;
        const int b_row = tn * BN + static_cast<int>(rank) * BN_CTA;
        for (int kb = 0; kb < p.num_k_blocks; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1u);
          const uint32_t sa = smem_u32(smem + stage * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
          uint32_t fb;
          if constexpr (CG == 1) {
            mbar_arrive_expect_tx(&full[stage], STAGE_BYTES);
            fb = smem_u32(&full[stage]);
          } else {
            if (rank == 0) mbar_arrive_expect_tx(&full[stage], 2 * STAGE_BYTES);
            fb = mapa_shared(smem_u32(&full[stage]), 0);
          }
          const int k0 = kb * BK;
          if constexpr (!A_MN) {
            if constexpr (CG == 1) tma_load_2d(&tmA, sa, fb, k0, a_row, pol);
            else tma_load_2d_pair(&tmA, sa, fb, k0, a_row, pol);
          } else {
#pragma unroll
            for (int h = 0; h < BM / 64; ++h) {
              if constexpr (CG == 1) tma_load_2d(&tmA, sa + h * 8192, fb, a_row + 64 * h, k0, pol);
              else tma_load_2d_pair(&tmA, sa + h * 8192, fb, a_row + 64 * h, k0, pol);
            }
          }
          if constexpr (!B_MN) {
            if constexpr (CG == 1) tma_load_2d(&tmB, sb, fb, k0, b_row, pol);
            else tma_load_2d_pair(&tmB, sb, fb, k0, b_row, pol);
          } else {
#pragma unroll
            for (int h = 0; h < BN_CTA / 64; ++h) {
              if constexpr (CG == 1) tma_load_2d(&tmB, sb + h * 8192, fb, b_row + 64 * h, k0, pol);
              else tma_load_2d_pair(&tmB, sb + h * 8192, fb, b_row + 64 * h, k0, pol);
            }
          }
          if (++stage == STAGES) { stage = 0; phase ^= 1u; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (leader CTA)
    if (rank == 0 && lane == 0) {
      uint32_t stage = 0, phase = 0;
      int it = 0;
      for (int t = cluster_id; t < num_tiles; t += num_clusters, ++it) {
        const uint32_t acc = it & 1;
        const uint32_t acc_phase = (it >> 1) & 1;
        if constexpr (CG == 2) mbar_wait_cluster(&tempty[acc], acc_phase ^ 1u);
        else mbar_wait(&tempty[acc], acc_phase ^ 1u);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < p.num_k_blocks; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + stage * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            const uint64_t ad = A_MN ? sdesc_mn_sw128(sa + k * A_KSTEP, 8192) : sdesc_k_sw128(sa + k * A_KSTEP);
            const uint64_t bd = B_MN ? sdesc_mn_sw128(sb + k * B_KSTEP, 8192) : sdesc_k_sw128(sb + k * B_KSTEP);
            umma_f16<CG>(d_tmem, ad, bd, IDESC, (kb | k) != 0 ? 1u : 0u);
          }
          umma_commit<CG>(&empty[stage]);  // frees the smem stage once these MMAs retire
          if (++stage == STAGES) { stage = 0; phase ^= 1u; }
        }
        umma_commit<CG>(&tfull[acc]);      // accumulator ready for the epilogue
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue warps
    const uint32_t quad = warp & 3u;
    const uint32_t tempty_addr = (CG == 2) ? mapa_shared(smem_u32(&tempty[0]), 0) : smem_u32(&tempty[0]);
    int it = 0;
    for (int t = cluster_id; t < num_tiles; t += num_clusters, ++it) {
      int tm, tn;
      tile_coords(t, p, tm, tn);
      const uint32_t acc = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = tm * BM * CG + static_cast<int>(rank) * BM + static_cast<int>(quad * 32 + lane);
      const int col0 = tn * BN;
      const uint32_t tbase = tmem_base + ((quad * 32u) << 16) + acc * BN;
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        uint32_t v[32];
        tmem_ld_32x32b_x32(tbase + c * 32, v);
        tmem_ld_wait();
        if (c == BN / 32 - 1) {
          // All TMEM reads of this accumulator are done: hand it back to the MMA warp.
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            if constexpr (CG == 2) mbar_arrive_cluster(tempty_addr + acc * 8);
            else mbar_arrive(&tempty[acc]);
          }
        }
        store_chunk<OUT_F32>(p, row, col0 + c * 32, v);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<CG>(tmem_base, S::TMEM_COLS);
  }
#endif
}

}  // namespace hg
