// HBM-streaming tcgen05 HGEMM for skinny shapes (BASELINE.json configs[3]:
// C = A B with m = 16384, n = 64..256, k = 4096, paper layout TN).
//
// Same kernel coordinates as hgemm_tc.cuh: D = C^T row-major (M = n, N = m,
// ldd = ldc), Ak = op(B)^T (M x K), Bk = op(A) (N x K), both K-major (TN).
// With M <= 256 the arithmetic intensity is <= ~M FLOP/B, at or below the
// B200 ridge: the time is the single pass over Bk (the m x k operand, 128 MiB
// at the config), so the kernel is shaped for HBM streaming, not for tensor
// throughput:
//   * persistent CTAs, one per SM; N is cut into chunks of CW columns with
//     CW (a multiple of 16, runtime) chosen so that the chunk count is a
//     multiple of the SM count -- every SM streams the same number of Bk rows
//     (tiles of 128/256 columns would leave 20 of 148 SMs idle at m = 16384);
//   * the ring depth is a runtime value: as many stages of (Ak 128 x 64 per
//     M-subtile, or 64 x 64 when M <= 64; L2-resident) + (Bk CW x 64, from
//     HBM) as fit in 227 KB, so each SM keeps 100-140 KB of Bk loads in flight
//     (Little's law; tools/stream_study.py measures the TMA streaming curve);
//   * MT = M-subtiles of 128 rows (M <= 128: 1, M <= 256: 2); one tcgen05.mma
//     M = 128, N = CW per subtile and K = 16 step (instruction descriptor N is
//     a runtime field); accumulators double-buffered in TMEM across chunks;
//   * epilogue: 4 warps, TMEM -> registers -> alpha*acc + beta*C (FP32) ->
//     FP16/FP32, stored straight to global (C is small: M x N).
// Paper mapping: Alg. 1 with the b_m x b_n block degenerated to
// M x CW; the paper's DRAM-bound analysis (SVI-A) is exactly this
// regime: with b_m = M small the intensity b_m b_n/(b_m + b_n) is
// bounded by M, so the only lever left is the memory system.
#pragma once
#include <cuda_fp16.h>

#include "hgemm_tc.cuh"
#include "ptx.cuh"

namespace hg {

struct StreamParams {
  int32_t M, N, K;        // D is M x N (M <= 128 * MT), reduction length K
  int32_t cw;             // chunk width along N: multiple of 16, 16..256/MT
  int32_t num_chunks;     // ceil(N / cw)
  int32_t num_k_blocks;   // ceil(K / 64)
  int32_t stages;         // ring depth (<= kStreamMaxStages)
  int32_t kg;             // k-blocks per stage (G); > 1 only with the 3-D Bk map (K % 64 == 0, G | nkb)
  uint32_t stage_bytes;   // G * (a_bytes + cw * 128), a multiple of 1024
  uint32_t a_bytes;       // Ak bytes per k-block: MT * 16 KB, or 8 KB when M <= 64 (see below)
  int32_t k_rot;          // 1: CTA c walks its k-blocks starting at c * nkb / gridDim (see below)
  float alpha, beta;
  void *D;
  int64_t ldd;
  unsigned long long *probe;  // HGEMM_TRACE builds: per-CTA %globaltimer events (tools/trace_stream.py)
  // 1: D is stored transposed, element (row, col) at D + col*ldd + row (the
  // swapped-operand use for small m: the kernel streams op(B) and keeps op(A)
  // resident, computing C = op(A) op(B) with C column-major; each warp's 32 rows
  // are consecutive in memory, so every column store is one 64/128-B segment)
  int32_t tout;
  // 1: tmB is the 3-D k-block-grouped view of Bk (dims {64, N, K/64}, strides
  // {ldb, 128 B}, box {64, cw, G}): one TMA load brings G k-blocks of every Bk
  // row, G x 128 contiguous bytes per row, in the smem image of G ordinary SW128
  // tiles.  The pure streaming study (tools/stream_study.py --3d) measures
  // 26.6 us instead of 28.7 us for 128 MiB at G >= 2 (5.04 vs 4.67 TB/s).
  int32_t b3d;
  int32_t pre;            // stage loads issued before the CTA barrier (1 .. stages)
  // 1: tmA is the 3-D k-group view of Ak too (MT == 1, kg == 2): the stage's two Ak k-blocks
  // (64 or 128 rows each) come from ONE load of 256 contiguous bytes per row (the TMA engine
  // is limited by row requests)
  int32_t a3d;
};

#ifdef HGEMM_TRACE
#define ST_TRACE(f)                                                                                  \
  do {                                                                                               \
    if (p.probe != nullptr) p.probe[8 * blockIdx.x + (f)] = globaltimer_ns();                        \
  } while (0)
#else
#define ST_TRACE(f) \
  do {              \
  } while (0)
#endif

constexpr int kStreamMaxStages = 16;
constexpr uint32_t kStreamSmemBytes = 227u * 1024u;

// Runtime instruction descriptor: kind::f16, D FP32, A/B FP16 K-major, M = 128, N = n.
__device__ __forceinline__ uint32_t idesc_f16_m128(uint32_t n) {
  return (1u << 4) | ((n >> 3) << 17) | ((128u >> 4) << 24);
}

__device__ __forceinline__ void tmem_ld_32x32b_x16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}

template <int MT, bool OUT_F32>
__global__ void __launch_bounds__(192, 1)
    hgemm_stream_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        const StreamParams p) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  constexpr uint32_t A_SUB = 128u * 64u * 2u;  // one 128-row Ak subtile of a k-block (16 KB)
  // M <= 64: the TMA box holds the 64 real Ak rows only (8 KB); the M = 128 MMA
  // then reads the next 8 KB of shared memory (the next Ak k-block, the stage's
  // Bk, the next stage or the pad behind the ring) as Ak rows 64..127, which
  // only feed accumulator lanes 64..127 -- rows >= M that are never stored.
  // One k-block shrinks from 30 to 22 KB (n = 64, cw = 112), 20 to 12 KB (m = 64, cw = 32).
  const uint32_t a_bytes = p.a_bytes;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw_u32 = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw_u32 & 1023u)) & 1023u);
  const int stages = p.stages;
  const uint32_t stage_bytes = p.stage_bytes;
  // M <= 64 (8 KB Ak boxes): the last Ak tile's MMA reads 8 KB past its box, so the
  // barriers sit behind an 8 KB pad after the ring (the host sizes the allocation)
  const uint32_t pad = a_bytes == 8192u ? 8192u : 0u;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + stages * stage_bytes + pad);
  uint64_t *empty = full + kStreamMaxStages;
  uint64_t *tfull = empty + kStreamMaxStages;  // [2]
  uint64_t *tempty = tfull + 2;                // [2]
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tempty + 2);

  const uint32_t warp = warp_id();
  const uint32_t lane = lane_id();
  if (threadIdx.x == 0) ST_TRACE(0);
  const int cw = p.cw;
  // k-block order: with k_rot, CTA c starts its k loop at c * nkb / gridDim and
  // wraps, so that at any moment the CTAs read different column offsets of
  // their op(A) rows (rows are K-contiguous, 2K bytes apart) instead of all
  // hitting the same offset in every row.  Only the summation order changes.
  const int nkb = p.num_k_blocks;
  // TMA producer state (warp 0, lane 0): iteration pi of chunk pch is loaded into stage pstage
  uint32_t pstage = 0, pphase = 0;
  int pch = blockIdx.x, pi = 0;
  // Stage layout: [G Ak k-blocks of a_bytes][G Bk k-blocks of cw * 128 B]
  const int kg = p.kg;
  const int ngr = nkb / kg;  // k-block groups (stages) per chunk
  const int gr_rot = p.k_rot ? static_cast<int>((static_cast<int64_t>(blockIdx.x) * ngr) / gridDim.x) : 0;
  const uint32_t b_off = static_cast<uint32_t>(kg) * a_bytes;
  const uint32_t b_kb = static_cast<uint32_t>(cw) * 128u;
  auto produce = [&](int max_loads) {  // issue up to max_loads more stage loads
    for (; pch < p.num_chunks && max_loads > 0; --max_loads) {
      const int kb0 = ((pi + gr_rot) % ngr) * kg;
      mbar_wait(&empty[pstage], pphase ^ 1u);
      const uint32_t sa = smem_u32(smem + pstage * stage_bytes);
      mbar_arrive_expect_tx(&full[pstage], stage_bytes);
      const uint32_t fb = smem_u32(&full[pstage]);
      if (MT == 1 && p.a3d) {
        tma_load_3d(&tmA, sa, fb, 0, 0, kb0);
      } else {
        for (int j = 0; j < kg; ++j) {
#pragma unroll
          for (int t = 0; t < MT; ++t) tma_load_2d(&tmA, sa + j * a_bytes + t * A_SUB, fb, (kb0 + j) * 64, t * 128, 0);
        }
      }
      if (p.b3d) tma_load_3d(&tmB, sa + b_off, fb, 0, pch * cw, kb0);
      else tma_load_2d(&tmB, sa + b_off, fb, kb0 * 64, pch * cw, 0);
      if (++pstage == static_cast<uint32_t>(stages)) { pstage = 0; pphase ^= 1u; }
      if (++pi == ngr) { pi = 0; pch += gridDim.x; }
    }
  };
  if (warp == 0 && lane == 0) {
    // The producer initialises the ring barriers itself and issues the first ring of
    // loads right away (after griddepcontrol.wait), so the first HBM round trip
    // overlaps the TMEM allocation and the CTA barrier below.
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    fence_mbarrier_init();
    griddep_wait();
    // p.pre (<= stages) stage loads before the CTA barrier: TMA issue stalls once the
    // engine's queue is full, and the MMA warp waits at the barrier behind it
    // (tools/trace_stream.py: with 16 stages issued here the first MMA started 5 us
    // after the kernel, 0.3 us after its data)
    produce(p.pre);
  }
  if (warp == 1) {
    if (lane == 0) {
      for (int b = 0; b < 2; ++b) {
        mbar_init(&tfull[b], 1);
        mbar_init(&tempty[b], 4);
      }
      fence_mbarrier_init();
    }
    __syncwarp();
    tmem_alloc<1>(smem_u32(tmem_slot), 512);
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  griddep_wait();  // PDL: the prologue overlapped the previous kernel
  if (threadIdx.x == 0) ST_TRACE(1);

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer (the remaining loads)
    if (lane == 0) produce(1 << 30);
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      const uint32_t idesc = idesc_f16_m128(static_cast<uint32_t>(cw));
      uint32_t stage = 0, phase = 0;
      int it = 0;
      for (int ch = blockIdx.x; ch < p.num_chunks; ch += gridDim.x, ++it) {
        const uint32_t buf = it & 1;
        const uint32_t acc_phase = (it >> 1) & 1;
        mbar_wait(&tempty[buf], acc_phase ^ 1u);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + buf * 256u;
        for (int g = 0; g < ngr; ++g) {  // iteration index (the smem stage holds group (g + gr_rot) % ngr)
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          if (it == 0 && g == 0) ST_TRACE(2);
          const uint32_t s0 = smem_u32(smem + stage * stage_bytes);
          for (int j = 0; j < kg; ++j) {
            const uint32_t sa = s0 + j * a_bytes;
            const uint32_t sb = s0 + b_off + j * b_kb;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t bd = sdesc_k_sw128(sb + k * 32);
#pragma unroll
              for (int t = 0; t < MT; ++t)
                umma_f16<1>(d_tmem + t * cw, sdesc_k_sw128(sa + t * A_SUB + k * 32), bd, idesc,
                            (g | j | k) != 0 ? 1u : 0u);
            }
          }
          umma_commit<1>(&empty[stage]);
          if (++stage == static_cast<uint32_t>(stages)) { stage = 0; phase ^= 1u; }
        }
        umma_commit<1>(&tfull[buf]);
        if (it == 0) ST_TRACE(3);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (warps 2..5)
    const uint32_t quad = warp & 3u;
    const float alpha = p.alpha, beta = p.beta;
    int it = 0;
    for (int ch = blockIdx.x; ch < p.num_chunks; ch += gridDim.x, ++it) {
      const uint32_t buf = it & 1;
      const uint32_t acc_phase = (it >> 1) & 1;
      if (lane == 0) mbar_wait(&tfull[buf], acc_phase);
      __syncwarp();
      tc_fence_after();
      if (warp == 2 && lane == 0 && it == 0) ST_TRACE(4);
      const int n0 = ch * cw;
#pragma unroll
      for (int t = 0; t < MT; ++t) {
        const int row = t * 128 + static_cast<int>(quad) * 32 + static_cast<int>(lane);
        const uint32_t tbase = tmem_base + ((quad * 32u) << 16) + buf * 256u + t * cw;
#pragma unroll 1
        for (int c = 0; c < cw; c += 16) {
          uint32_t v[16];
          tmem_ld_32x32b_x16(tbase + c, v);
          tmem_ld_wait();
          const int col = n0 + c;
          if (row >= p.M || col >= p.N) continue;
          float r[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) r[j] = alpha * __uint_as_float(v[j]);
          if (p.tout) {  // transposed D: column col+j is contiguous over this warp's rows
            const int nj = min(16, p.N - col);
            if (beta != 0.0f) {  // all 16 C loads first (no store in between), then the stores
              float cv[16];
#pragma unroll
              for (int j = 0; j < 16; ++j) {
                const int64_t o = static_cast<int64_t>(col + j) * p.ldd + row;
                if constexpr (OUT_F32) cv[j] = j < nj ? static_cast<const float *>(p.D)[o] : 0.0f;
                else cv[j] = j < nj ? __half2float(static_cast<const __half *>(p.D)[o]) : 0.0f;
              }
#pragma unroll
              for (int j = 0; j < 16; ++j) r[j] = fmaf(beta, cv[j], r[j]);
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) {
              if (j >= nj) break;
              const int64_t o = static_cast<int64_t>(col + j) * p.ldd + row;
              if constexpr (OUT_F32) static_cast<float *>(p.D)[o] = r[j];
              else static_cast<__half *>(p.D)[o] = __float2half_rn(r[j]);
            }
            continue;
          }
          const int64_t off = static_cast<int64_t>(row) * p.ldd + col;
          const bool whole = col + 16 <= p.N;  // 16 columns inside N: 16-B aligned vectors
          if constexpr (OUT_F32) {
            float *dst = static_cast<float *>(p.D) + off;
            if (whole) {
              if (beta != 0.0f) {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                  const float4 cv = reinterpret_cast<const float4 *>(dst)[q];
                  r[4 * q] = fmaf(beta, cv.x, r[4 * q]);
                  r[4 * q + 1] = fmaf(beta, cv.y, r[4 * q + 1]);
                  r[4 * q + 2] = fmaf(beta, cv.z, r[4 * q + 2]);
                  r[4 * q + 3] = fmaf(beta, cv.w, r[4 * q + 3]);
                }
              }
#pragma unroll
              for (int q = 0; q < 4; ++q)
                reinterpret_cast<float4 *>(dst)[q] = make_float4(r[4 * q], r[4 * q + 1], r[4 * q + 2], r[4 * q + 3]);
            } else {
#pragma unroll
              for (int j = 0; j < 16; ++j)
                if (col + j < p.N) dst[j] = beta != 0.0f ? fmaf(beta, dst[j], r[j]) : r[j];
            }
          } else {
            __half *dst = static_cast<__half *>(p.D) + off;
            if (whole) {
              uint32_t w[8];
              if (beta != 0.0f) {
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                  const uint4 cv = reinterpret_cast<const uint4 *>(dst)[q];
                  const uint32_t cw4[4] = {cv.x, cv.y, cv.z, cv.w};
#pragma unroll
                  for (int e = 0; e < 4; ++e) {
                    const float2 cf = __half22float2(*reinterpret_cast<const __half2 *>(&cw4[e]));
                    const int j = 4 * q + e;
                    w[j] = pack_half2(fmaf(beta, cf.x, r[2 * j]), fmaf(beta, cf.y, r[2 * j + 1]));
                  }
                }
              } else {
#pragma unroll
                for (int j = 0; j < 8; ++j) w[j] = pack_half2(r[2 * j], r[2 * j + 1]);
              }
              reinterpret_cast<uint4 *>(dst)[0] = make_uint4(w[0], w[1], w[2], w[3]);
              reinterpret_cast<uint4 *>(dst)[1] = make_uint4(w[4], w[5], w[6], w[7]);
            } else {
#pragma unroll
              for (int j = 0; j < 16; ++j)
                if (col + j < p.N)
                  dst[j] = __float2half_rn(beta != 0.0f ? fmaf(beta, __half2float(dst[j]), r[j]) : r[j]);
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[buf]);
      if (warp == 2 && lane == 0 && it == 0) ST_TRACE(5);
    }
  }

  __syncwarp();  // reconverge the single-lane roles before the .aligned CTA barrier
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) ST_TRACE(6);
#ifdef HGEMM_TRACE
  if (threadIdx.x == 0 && p.probe != nullptr) {  // slot 7: the SM this CTA ran on
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    p.probe[8 * blockIdx.x + 7] = smid;
  }
#endif
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<1>(tmem_base, 512);
  }
#endif
}

}  // namespace hg
