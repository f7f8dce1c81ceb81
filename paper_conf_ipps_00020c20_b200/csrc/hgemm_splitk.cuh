// Split-K tcgen05 HGEMM for under-filled shapes.
//
// Same kernel coordinates as hgemm_tc.cuh (D = C^T row-major, Ak = op(B)^T,
// Bk = op(A)).  A cluster of S CTAs computes ONE 128 x BN output tile; CTA r
// of the cluster accumulates k-blocks [r*nkb/S, (r+1)*nkb/S) with
// tcgen05.mma (cta_group::1) into its own TMEM.  The S partial accumulators
// are then reduced through distributed shared memory, deterministically:
// CTA r owns the column slice [r*BN/S, (r+1)*BN/S); every CTA stages the
// slices of its FP32 partial it does not own in its (then idle) smem ring and
// sends each warp's 32 rows of a slice to the owner with ONE bulk copy
// (cp.async.bulk shared::cta -> shared::cluster) that completes on the owner's
// receive mbarrier; each owner waits for its (S-1) x 128 x BN/S FP32 values,
// sums the S slices in split order 0..S-1 (its own from registers; fixed
// order => run-to-run bitwise reproducible), applies alpha/beta and stores its
// slice of D.  No global workspace, no atomics, no cluster barrier between
// the mainloop and the reduction (the first version pushed 16-B remote stores
// and synchronised the cluster: 2.4 us from the last MMA to the reduction on
// the LSTM-gate shapes, profiles/r01b/trace_splitk_lstm.log).
//
// Paper mapping: the blocked algorithm of Alg. 1 with the K loop
// (line 6) divided among S thread blocks; the grid of SVI-A.2 is
// multiplied by S so that shapes with few output tiles (small-batch LSTM
// gates) still occupy the 148 SMs.
#pragma once
#include <cuda_fp16.h>

#include "hgemm_tc.cuh"
#include "ptx.cuh"

namespace hg {

// HM (half M): tiles of 64 valid Ak rows.  The TMA brings 64 rows (8 KB per k-block); the
// M = 128 MMA reads the next 8 KB of the same stage as rows 64..127 (the next Ak k-block or
// the stage's Bk), which only feed accumulator lanes 64..127 -- never read.  Twice the tiles for the same K split: the LSTM
// gates at batch 64 run 64 tiles x 2 splits instead of 32 x 4 (a 2-way reduction).
template <int BN, int S, bool HM = false>
struct SkShape {
  static constexpr int BM = HM ? 64 : 128;                 // valid tile rows
  static constexpr int BK = 64;
  static constexpr uint32_t A_BYTES = BM * BK * 2;         // Ak bytes loaded per k-block
  static constexpr uint32_t B_BYTES = BN * BK * 2;
  static constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  // receive buffer: (S-1) peer slots x 128 rows x BN/S FP32 (peer src lands in slot
  // src < rank ? src : src - 1; the owner's own slice stays in registers)
  static constexpr uint32_t PART_BYTES = (S - 1) * BM * (BN / S) * 4;
  static constexpr int STAGES_FIT = static_cast<int>((227u * 1024u - PART_BYTES - 2048u) / STAGE_BYTES);
  // At most 6 stages: 8 for BN = 64 (every k-block of an LSTM-gate CTA in flight at once) fit
  // but measured 0.9 us slower per launch (profiles/r02/splitk_stages_sweep.log)
  static constexpr int STAGES = STAGES_FIT > 6 ? 6 : STAGES_FIT;
  static constexpr uint32_t TMEM_COLS = BN < 32 ? 32 : BN;
  static constexpr uint32_t SMEM_BYTES = STAGES * STAGE_BYTES + PART_BYTES + 1024 + 1024;
  static constexpr int SLICE = BN / S;                     // output columns reduced by each CTA
  static_assert(BN == 64 || BN == 128, "BN");
  static_assert(S == 2 || S == 4 || S == 8, "S");
  static_assert(SLICE % 8 == 0, "slice");
  static_assert(STAGES >= 2, "stages");
  static_assert(BM * BN * 4 <= STAGES * STAGE_BYTES, "reduction staging ([owner][row][SLICE]) in the smem ring");
};

// Receive buffer of the owner CTA: [S-1 peer slots][128 rows][SLICE FP32] (the
// sender stages in the same layout with S owner slots), the
// 16-byte chunk index of a row rotated by the row so that consecutive rows
// (threads) writing or reading the same chunk use different bank groups.
template <int SLICE, int ROWS = 128>
__device__ __forceinline__ uint32_t recv_off_t(uint32_t src, uint32_t row, uint32_t chunk) {
  constexpr uint32_t CH = SLICE / 4;                      // 16-byte chunks per row
  // 16-B accesses go to shared memory in phases of 8 lanes (rows): the 8 rows of a phase
  // must cover the 8 16-B bank groups.  Rows are CH chunks apart, so consecutive rows repeat
  // the bank group every 8/CH rows when CH < 8: rotate by row / (8/CH) then.
  constexpr uint32_t D = CH >= 8 ? 1u : 8u / CH;
  const uint32_t q = (chunk + row / D) % CH;
  return (src * static_cast<uint32_t>(ROWS) + row) * (SLICE * 4u) + q * 16u;
}

// NC consecutive TMEM columns of this thread's lane (32x32b shape), NC = 8, 16, 32 or 64.
template <int NC>
__device__ __forceinline__ void sk_tmem_ld(uint32_t taddr, uint32_t *r) {
  if constexpr (NC == 8) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
  } else if constexpr (NC == 16) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
        "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
  } else {
#pragma unroll
    for (int c = 0; c < NC / 32; ++c)
      tmem_ld_32x32b_x32(taddr + c * 32, *reinterpret_cast<uint32_t(*)[32]>(r + 32 * c));
  }
}

// 16 bytes from registers into a peer CTA's shared memory, completing 16 bytes of
// transaction count on the peer's mbarrier (both shared::cluster addresses).
__device__ __forceinline__ void st_async_v4(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d,
                                            uint32_t mbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];"
               ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d), "r"(mbar)
               : "memory");
}

__device__ __forceinline__ void st_shared_cluster_v4(uint32_t addr, uint32_t a, uint32_t b, uint32_t c,
                                                     uint32_t d) {
  asm volatile("st.shared::cluster.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d)
               : "memory");
}
__device__ __forceinline__ float4 ld_shared_f4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr)
               : "memory");
  return v;
}

__device__ __forceinline__ float4 ld_shared_cluster_v4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(addr)
               : "memory");
  return v;
}

template <int BN, int S, bool A_MN, bool B_MN, bool OUT_F32, bool HM = false>
__global__ void __launch_bounds__(192, 1)
    hgemm_splitk_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        const TcParams p) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  using SH = SkShape<BN, S, HM>;
  constexpr int BM = SH::BM;
  constexpr int BK = SH::BK;
  constexpr int STAGES = SH::STAGES;
  constexpr uint32_t A_BYTES = SH::A_BYTES;
  constexpr uint32_t STAGE_BYTES = SH::STAGE_BYTES;
  constexpr uint32_t IDESC = make_idesc_f16<128, BN, A_MN, B_MN>();  // M = 128 (HM: 64 valid rows)
  constexpr uint32_t A_KSTEP = A_MN ? 16 * 128 : 32;
  constexpr uint32_t B_KSTEP = B_MN ? 16 * 128 : 32;

  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw_u32 = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw_u32 & 1023u)) & 1023u);
  uint8_t *part = smem + STAGES * STAGE_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(part + SH::PART_BYTES);
  uint64_t *empty = full + STAGES;
  uint64_t *tfull = empty + STAGES;
  uint64_t *rbar = tfull + 1;  // receive barrier: (S-1) slices of 128 x SLICE FP32 from the peers
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(rbar + 1);

  const uint32_t warp = warp_id();
  const uint32_t lane = lane_id();
  const uint32_t rank = cluster_ctarank();
  const int tile = static_cast<int>(blockIdx.x) / S;
  int tm, tn;
  tile_coords(tile, p, tm, tn);
  const int kb0 = static_cast<int>((static_cast<int64_t>(p.num_k_blocks) * rank) / S);
  const int kb1 = static_cast<int>((static_cast<int64_t>(p.num_k_blocks) * (rank + 1)) / S);
  const int nkb = kb1 - kb0;
  auto recv_off = [](uint32_t src, uint32_t row, uint32_t chunk) { return recv_off_t<SH::SLICE, BM>(src, row, chunk); };

#ifdef HGEMM_TRACE
#define SK_TRACE(f)                                                                            \
  do {                                                                                         \
    if (p.probe != nullptr && blockIdx.x < 256) p.probe[8 + 8 * blockIdx.x + (f)] = globaltimer_ns(); \
  } while (0)
// prologue detail (second region): p.probe[8 + 2048 + 8*blockIdx.x + f]
#define SK_TRACE2(f)                                                                           \
  do {                                                                                         \
    if (p.probe != nullptr && blockIdx.x < 256) p.probe[8 + 2048 + 8 * blockIdx.x + (f)] = globaltimer_ns(); \
  } while (0)
#define SK_TRACE3(f)                                                                           \
  do {                                                                                         \
    if (p.probe != nullptr && blockIdx.x < 256) p.probe[8 + 4096 + 8 * blockIdx.x + (f)] = globaltimer_ns(); \
  } while (0)
#else
#define SK_TRACE3(f) \
  do {               \
  } while (0)
#define SK_TRACE(f) \
  do {              \
  } while (0)
#define SK_TRACE2(f) \
  do {               \
  } while (0)
#endif
  if (threadIdx.x == 0) SK_TRACE(0);
  // TMA producer state (warp 0, lane 0): k-block pkb is loaded into ring stage pstage
  const int a_row = tm * BM;
  const int b_row = tn * BN;
  // k-groups (p.sk_kg = G = 1 or 2, the host guarantees G | nkb): a ring stage holds G
  // consecutive k-blocks, [G Ak k-blocks][G Bk k-blocks]; with G = 2 the Ak k-blocks come
  // from ONE 3-D TMA load (tmA = the k-group view, box {64, 128, 2}), 256 contiguous bytes
  // per Ak row (HBM streaming).  The ring keeps its size:
  // STAGES / G stages of G * STAGE_BYTES.
  const int kg = (!A_MN && p.sk_kg == 2) ? 2 : 1;
  const int nst = STAGES / kg;
  const uint32_t sst_bytes = static_cast<uint32_t>(kg) * STAGE_BYTES;
  uint32_t pstage = 0, pphase = 0;
  int pkb = kb0;
  auto produce = [&](int upto) {  // issue the loads of k-blocks [pkb, upto), G per stage
    for (; pkb < upto; pkb += kg) {
      mbar_wait(&empty[pstage], pphase ^ 1u);
      const uint32_t sa = smem_u32(smem + pstage * sst_bytes);
      const uint32_t sb = sa + kg * A_BYTES;
      mbar_arrive_expect_tx(&full[pstage], sst_bytes);
      const uint32_t fb = smem_u32(&full[pstage]);
      const int k0 = pkb * BK;
      if constexpr (!A_MN) {
        if (kg == 2) tma_load_3d(&tmA, sa, fb, 0, a_row, pkb);
        else tma_load_2d(&tmA, sa, fb, k0, a_row, 0);
      } else {
#pragma unroll
        for (int q = 0; q < BM / 64; ++q) tma_load_2d(&tmA, sa + q * 8192, fb, a_row + 64 * q, k0, 0);
      }
      if (!B_MN && kg == 2 && p.sk_b3d) {  // both Bk k-blocks of the stage: one 3-D box, 256 B per row
        tma_load_3d(&tmB, sb, fb, 0, b_row, pkb);
      } else for (int j = 0; j < kg; ++j) {
        if constexpr (!B_MN) {
          tma_load_2d(&tmB, sb + j * SH::B_BYTES, fb, k0 + j * BK, b_row, 0);
        } else {
#pragma unroll
          for (int q = 0; q < BN / 64; ++q)
            tma_load_2d(&tmB, sb + j * SH::B_BYTES + q * 8192, fb, b_row + 64 * q, k0 + j * BK, 0);
        }
      }
#ifdef HGEMM_TRACE
      if (pkb == kb0) SK_TRACE2(6);
#endif
      if (++pstage == static_cast<uint32_t>(nst)) { pstage = 0; pphase ^= 1u; }
    }
  };
  if (warp == 0 && lane == 0) {
    // The producer initialises the ring barriers itself and issues the first ring of
    // loads right away (after griddepcontrol.wait), so the first HBM round trip
    // overlaps the TMEM allocation and the CTA barrier below.
    SK_TRACE2(0);
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int s = 0; s < nst; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    fence_mbarrier_init();
    SK_TRACE2(1);
    griddep_wait();
    SK_TRACE2(2);
    produce(min(kb1, kb0 + nst * kg));
    SK_TRACE2(3);
  }
  if (warp == 1) {
    if (lane == 0) {
      mbar_init(tfull, 1);
      mbar_init(rbar, 1);
      // the peers' bulk copies complete their bytes on rbar (possibly before this arrival:
      // the transaction count may run negative until the expectation is registered)
      mbar_arrive_expect_tx(rbar, (S - 1) * static_cast<uint32_t>(BM) * SH::SLICE * 4u);
      fence_mbarrier_init();
    }
    __syncwarp();
    if (lane == 0) SK_TRACE2(4);
    tmem_alloc<1>(smem_u32(tmem_slot), SH::TMEM_COLS);
    if (lane == 0) SK_TRACE2(5);
  }
  __syncwarp();
  if (lane == 0 && warp == 2) SK_TRACE3(0);
  if (lane == 0 && warp == 5) SK_TRACE3(1);
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) SK_TRACE3(2);
  tc_fence_after();
  // Cluster barrier, split: every thread arrives now (its barriers are initialised); a
  // thread waits only before its first access to a peer's shared memory (the epilogue's
  // bulk copies) or, for the producer / MMA warps, before exiting.
  cluster_arrive();
  const uint32_t tmem_base = *tmem_slot;
  if (threadIdx.x == 0) SK_TRACE(1);
  griddep_wait();  // PDL: the prologue above overlapped the previous kernel; C is read right below
  // Epilogue warps prefetch their C slice (FP16 vector path, beta != 0) at
  // kernel start: C does not depend on the accumulator.
  uint32_t cpre[SH::SLICE / 2];
#pragma unroll
  for (int j = 0; j < SH::SLICE / 2; ++j) cpre[j] = 0u;
  if constexpr (!OUT_F32) {
    if (warp >= 2 && p.beta != 0.0f) {
      const int row = tm * BM + static_cast<int>((warp & 3u) * 32u + lane);
      const int col0 = tn * BN + static_cast<int>(rank) * SH::SLICE;
      if ((warp & 3u) * 32u < static_cast<uint32_t>(BM) && row < p.M && col0 + SH::SLICE <= p.N && (p.ldd & 7) == 0) {
        const uint4 *src = reinterpret_cast<const uint4 *>(static_cast<const __half *>(p.D) +
                                                          static_cast<int64_t>(row) * p.ldd + col0);
#pragma unroll
        for (int q = 0; q < SH::SLICE / 8; ++q) {
          const uint4 v = src[q];
          cpre[4 * q] = v.x;
          cpre[4 * q + 1] = v.y;
          cpre[4 * q + 2] = v.z;
          cpre[4 * q + 3] = v.w;
        }
      }
    }
  }
  if (lane == 0 && warp == 2) SK_TRACE3(3);

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer (the rest of the k range)
    if (lane == 0) produce(kb1);
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      uint32_t stage = 0, phase = 0;
      for (int j = 0; j < nkb; j += kg) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (j == 0) SK_TRACE(2);
        const uint32_t s0 = smem_u32(smem + stage * sst_bytes);
        for (int jj = 0; jj < kg; ++jj) {
          const uint32_t sa = s0 + jj * A_BYTES;
          const uint32_t sb = s0 + kg * A_BYTES + jj * SH::B_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            const uint32_t a_addr = sa + k * A_KSTEP;
            const uint32_t b_addr = sb + k * B_KSTEP;
            const uint64_t ad = A_MN ? sdesc_mn_sw128(a_addr, 8192) : sdesc_k_sw128(a_addr);
            const uint64_t bd = B_MN ? sdesc_mn_sw128(b_addr, 8192) : sdesc_k_sw128(b_addr);
            umma_f16<1>(tmem_base, ad, bd, IDESC, (j | jj | k) != 0 ? 1u : 0u);
          }
        }
        umma_commit<1>(&empty[stage]);
        if (++stage == static_cast<uint32_t>(nst)) { stage = 0; phase ^= 1u; }
      }
      SK_TRACE(3);
      if (nkb > 0) umma_commit<1>(tfull);
      else mbar_arrive(tfull);  // empty K range: the partial is zero
    }
  } else {
    // ------------------------------------------------------------ epilogue warps: split-K reduction
    // CTA `rank` owns output columns [rank*SLICE, (rank+1)*SLICE) of the tile.  Each
    // thread holds one tile row (its TMEM lane).  The slices owned by the peers are
    // staged in the smem ring (free: every MMA has retired and no load is pending)
    // in the owner's receive layout, then each warp sends its 32 rows of slice o with
    // one bulk copy to owner o's buffer [rank][rows], completing on o's rbar.
    constexpr int SLICE = SH::SLICE;
    constexpr uint32_t SLAB = static_cast<uint32_t>(BM) * SLICE * 4u;  // one source's slice block: BM rows x SLICE FP32
    const uint32_t quad = warp & 3u;
    const uint32_t prow = quad * 32u + lane;  // TMEM lane == tile row
    const bool act = quad * 32u < static_cast<uint32_t>(BM);  // HM: the warps of lanes 64..127 hold no valid rows
    const uint32_t stg = smem_u32(smem);      // staging: [owner][row][SLICE] (recv_off layout)
    float own[SLICE];
    // exp_flags & 64 (experiment): push each 16-B chunk of a peer's slice straight from
    // registers into the owner's receive buffer (st.async, completing on its rbar) instead
    // of staging the slices locally and sending them with bulk copies
    const bool direct = (p.exp_flags & 64) != 0;
    // Every peer's rbar is initialised before we copy / store into it: the cluster barrier's
    // wait phase, taken here while the mainloop runs (all CTAs arrived in their prologues).
    cluster_wait();
    const uint32_t part_u32 = smem_u32(part), rbar_u32 = smem_u32(rbar);
    mbar_wait(tfull, 0);
    tc_fence_after();
    if (warp == 2 && lane == 0) SK_TRACE(4);
    // Slice t of this row is owned by CTA (rank + t) % S; t = 0 is this CTA's own slice.  The
    // TMEM column offset of a slice is a runtime value (the rank), so each slice is one TMEM
    // load and its chunk offsets in the receive layout are per-thread constants: no per-chunk
    // branching on the owner (the unrolled per-column version executed ~500 instructions per
    // thread here).
    uint32_t qoff[SLICE / 4];  // this row's 16-B chunk q inside a slice block (recv_off swizzle)
#pragma unroll
    for (int q = 0; q < SLICE / 4; ++q) qoff[q] = recv_off(0u, prow, static_cast<uint32_t>(q));
    if (act) {
      uint32_t w[S][SLICE];
      if (nkb > 0) {
#pragma unroll
        for (int t = 0; t < S; ++t)
          sk_tmem_ld<SLICE>(tmem_base + ((quad * 32u) << 16) + ((rank + t) & (S - 1)) * SLICE, w[t]);
        tmem_ld_wait();
        if (warp == 2 && lane == 0) SK_TRACE3(4);
      } else {
#pragma unroll
        for (int t = 0; t < S; ++t)
#pragma unroll
          for (int j = 0; j < SLICE; ++j) w[t][j] = 0u;
      }
#pragma unroll
      for (int j = 0; j < SLICE; ++j) own[j] = __uint_as_float(w[0][j]);
#pragma unroll
      for (int t = 1; t < S; ++t) {
        const uint32_t owner = (rank + t) & (S - 1);
        if (direct) {
          const uint32_t slot = rank < owner ? rank : rank - 1u;
          const uint32_t rbase = mapa_shared(part_u32 + slot * SLAB, owner), rb = mapa_shared(rbar_u32, owner);
#pragma unroll
          for (int q = 0; q < SLICE / 4; ++q)
            st_async_v4(rbase + qoff[q], w[t][4 * q], w[t][4 * q + 1], w[t][4 * q + 2], w[t][4 * q + 3], rb);
        } else {
          const uint32_t base = stg + owner * SLAB;
#pragma unroll
          for (int q = 0; q < SLICE / 4; ++q)
            st_shared_v4(base + qoff[q], w[t][4 * q], w[t][4 * q + 1], w[t][4 * q + 2], w[t][4 * q + 3]);
        }
      }
    }
    if (warp == 2 && lane == 0) SK_TRACE3(5);
    tc_fence_before();
    if (!direct) {
      fence_proxy_async_smem();  // the staged slices -> the bulk copies (async proxy)
      __syncwarp();
    }
    if (lane == 0 && !direct && act) {
      const uint32_t rows_off = quad * 32u * SLICE * 4u;  // this warp's 32 rows in a slice block
#pragma unroll 1
      for (uint32_t o = 0; o < static_cast<uint32_t>(S); ++o) {
        if (o == rank) continue;
        const uint32_t slot = rank < o ? rank : rank - 1u;  // this CTA's slot in owner o's buffer
        bulk_copy_s2cluster(mapa_shared(smem_u32(part) + slot * SLAB + rows_off, o), stg + o * SLAB + rows_off,
                            32u * SLICE * 4u, mapa_shared(smem_u32(rbar), o));
      }
    }
    if (warp == 2 && lane == 0) SK_TRACE(5);

    // ------------------------------------------------------------ reduce + epilogue of this CTA's slice
    const int row = tm * BM + static_cast<int>(prow);
    const int col0 = tn * BN + static_cast<int>(rank) * SLICE;
    const uint32_t rbuf = smem_u32(part);
    if (S > 1 && act) mbar_wait(rbar, 0);  // the (S-1) peers' slices have landed
    if (warp == 2 && lane == 0) SK_TRACE3(6);
    float acc[SLICE];
#pragma unroll
    for (int j = 0; j < SLICE; ++j) acc[j] = 0.0f;
#pragma unroll
    for (int src = 0; src < (act ? S : 0); ++src) {  // fixed summation order: split 0, 1, ..., S-1
      if (static_cast<uint32_t>(src) == rank) {
#pragma unroll
        for (int j = 0; j < SLICE; ++j) acc[j] += own[j];
        continue;
      }
      const uint32_t slot = static_cast<uint32_t>(src) < rank ? static_cast<uint32_t>(src) : static_cast<uint32_t>(src) - 1u;
      const uint32_t sbase = rbuf + slot * SLAB;
#pragma unroll
      for (int q = 0; q < SLICE / 4; ++q) {
        const float4 v = ld_shared_f4(sbase + qoff[q]);
        acc[4 * q + 0] += v.x;
        acc[4 * q + 1] += v.y;
        acc[4 * q + 2] += v.z;
        acc[4 * q + 3] += v.w;
      }
    }
    if (warp == 2 && lane == 0) SK_TRACE3(7);
    if (act && row < p.M) {
      const float alpha = p.alpha, beta = p.beta;
      if constexpr (OUT_F32) {
        float *dst = static_cast<float *>(p.D) + static_cast<int64_t>(row) * p.ldd + col0;
#pragma unroll
        for (int j = 0; j < SLICE; ++j) {
          if (col0 + j < p.N) {
            float o = alpha * acc[j];
            if (beta != 0.0f) o = fmaf(beta, dst[j], o);
            dst[j] = o;
          }
        }
      } else {
        __half *dst = static_cast<__half *>(p.D) + static_cast<int64_t>(row) * p.ldd + col0;
        const bool vec = (col0 + SLICE <= p.N) && ((p.ldd & 7) == 0);
        if (vec) {
#pragma unroll
          for (int q = 0; q < SLICE / 8; ++q) {
            float f[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) f[e] = alpha * acc[8 * q + e];
            if (beta != 0.0f) {
              const __half2 *ch = reinterpret_cast<const __half2 *>(&cpre[4 * q]);
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
            reinterpret_cast<uint4 *>(dst)[q] = o;
          }
        } else {
#pragma unroll
          for (int j = 0; j < SLICE; ++j) {
            if (col0 + j < p.N) {
              float o = alpha * acc[j];
              if (beta != 0.0f) o = fmaf(beta, __half2float(dst[j]), o);
              dst[j] = __float2half_rn(o);
            }
          }
        }
      }
    }
  }

  if (threadIdx.x == 64) SK_TRACE(6);
  __syncwarp();
  if (warp < 2) cluster_wait();  // the producer / MMA warps' wait of the first cluster-barrier phase
  // Second phase: a CTA may exit only after its peers have received its slices (the
  // bulk copies read this CTA's staging area and complete only on the peers' rbar).
  cluster_sync();
  if (threadIdx.x == 0) SK_TRACE(7);
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<1>(tmem_base, SH::TMEM_COLS);
  }
#endif
}

}  // namespace hg
