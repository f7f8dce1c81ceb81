// B200 (sm_100a) micro-benchmarks: the paper's SIV-SV characterisation
// ("demystifying" the tensor core and the memory hierarchy, PAPER.md
// P:156-238, Tables I-V) redone for the units the tcgen05 HGEMM uses
// (SURVEY 8(f) NEXT-4).  Separate library (libhgemm_mb.so), not on the
// GEMM path; driven by tools/microbench.py.
//
//   mb_mma_rate   : tcgen05.mma kind::f16 issue-to-completion throughput
//                   (cycles per instruction) for cta_group::1 M=128 and
//                   cta_group::2 M=256, N in {64,128,256}; the analogue of
//                   Table I's HMMA.1688 CPI.
//   mb_mma_latency: one tcgen05.mma + tcgen05.commit -> mbarrier round trip.
//   mb_tmem_ld    : tcgen05.ld 32x32b.x32 bytes/cycle per SM with 4 or 8 warps.
//   mb_tma_load   : TMA (cp.async.bulk.tensor) bytes/cycle per SM and chip
//                   GB/s, from an L2-resident tile and streaming from HBM;
//                   the analogue of Table II / Table III.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "ptx.cuh"
#include "hgemm_tc.cuh"

namespace mb {
using namespace hg;

// ------------------------------------------------------------------ MMA throughput / latency
template <int CG, int N>
__global__ void __launch_bounds__(128, 1) mma_rate_kernel(int iters, unsigned long long *out, int latency_mode) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  constexpr int M = 128 * CG;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw & 1023u)) & 1023u);
  // operands: A 128 x 64 FP16 (16 KB) and B (N/CG) x 64 FP16, K-major SW128; contents irrelevant
  uint64_t *bar = reinterpret_cast<uint64_t *>(smem + 16384 + (N / CG) * 128);
  uint32_t *slot = reinterpret_cast<uint32_t *>(bar + 1);
  const uint32_t warp = warp_id(), lane = lane_id();
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0u;
  if (warp == 0) {
    if (lane == 0) {
      mbar_init(bar, 1);
      fence_mbarrier_init();
    }
    __syncwarp();
    tmem_alloc<CG>(smem_u32(slot), 512);
  }
  tc_fence_before();
  if constexpr (CG == 2) cluster_sync(); else __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *slot;
  constexpr uint32_t IDESC = make_idesc_f16<M, N, false, false>();
  if (warp == 0 && lane == 0 && rank == 0) {
    const uint32_t sa = smem_u32(smem), sb = sa + 16384;
    uint32_t phase = 0;
    long long t0 = clock64();
    if (!latency_mode) {
      for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < 4; ++k)
          umma_f16<CG>(tmem, sdesc_k_sw128(sa + 32 * k), sdesc_k_sw128(sb + 32 * k), IDESC, 1u);
      }
      umma_commit<CG>(bar);
      mbar_wait(bar, 0);
    } else {
      for (int i = 0; i < iters; ++i) {
        umma_f16<CG>(tmem, sdesc_k_sw128(sa), sdesc_k_sw128(sb), IDESC, 1u);
        umma_commit<CG>(bar);
        mbar_wait(bar, phase);
        phase ^= 1u;
      }
    }
    long long t1 = clock64();
    out[blockIdx.x] = static_cast<unsigned long long>(t1 - t0);
  }
  tc_fence_before();
  if constexpr (CG == 2) cluster_sync(); else __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc<CG>(tmem, 512);
  }
#endif
}

// ------------------------------------------------------------------ TMEM load bandwidth
__global__ void __launch_bounds__(256, 1) tmem_ld_kernel(int iters, int warps, int unroll, unsigned long long *out) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  __shared__ uint32_t slot;
  const uint32_t warp = warp_id(), lane = lane_id();
  if (warp == 0) tmem_alloc<1>(smem_u32(&slot), 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot;
  unsigned long long sink = 0;
  __syncthreads();
  long long t0 = clock64();
  if (warp < static_cast<uint32_t>(warps)) {
    const uint32_t base = tmem + (((warp & 3u) * 32u) << 16) + (warp >> 2) * 256u;
    if (unroll == 1) {
      for (int i = 0; i < iters; ++i) {
        uint32_t v[32];
        tmem_ld_32x32b_x32(base + (i & 7) * 32, v);
        tmem_ld_wait();
#pragma unroll
        for (int j = 0; j < 32; ++j) sink += v[j];
      }
    } else {
      for (int i = 0; i < iters; i += 4) {
        uint32_t v0[32], v1[32], v2[32], v3[32];
        tmem_ld_32x32b_x32(base + 0, v0);
        tmem_ld_32x32b_x32(base + 32, v1);
        tmem_ld_32x32b_x32(base + 64, v2);
        tmem_ld_32x32b_x32(base + 96, v3);
        tmem_ld_wait();
#pragma unroll
        for (int j = 0; j < 32; ++j) sink += v0[j] + v1[j] + v2[j] + v3[j];
      }
    }
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = static_cast<unsigned long long>(t1 - t0);
  if (sink == 0x123456789ull) out[gridDim.x] = sink;
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc<1>(tmem, 512);
  }
#endif
}

// ------------------------------------------------------------------ TMA load bandwidth
// One thread per CTA streams `iters` 128-row x 128-B boxes (16 KB) through a
// ring of 8 stages.  stride_rows = 0 re-reads the same tile (L2 resident);
// otherwise each CTA walks its own region of the tensor (HBM streaming).
__global__ void __launch_bounds__(32, 1) tma_load_kernel(const __grid_constant__ CUtensorMap tm, int iters,
                                                          int rows_total, int streaming, unsigned long long *out) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw & 1023u)) & 1023u);
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + 8 * 16384);
  if (threadIdx.x == 0) {
    for (int s = 0; s < 8; ++s) mbar_init(&full[s], 1);
    fence_mbarrier_init();
  }
  __syncwarp();
  if (threadIdx.x == 0) {
    const int boxes_per_row = 8;  // 8 boxes of 64 FP16 across a 512-element row band
    long long t0 = clock64();
    uint32_t phase = 0;
    for (int i = 0; i < iters + 8; ++i) {
      const int s = i & 7;
      if (i >= 8) {
        mbar_wait(&full[s], phase);
        if (s == 7) phase ^= 1u;
      }
      if (i < iters) {
        int row = 0, col = 0;
        if (streaming) {
          const int64_t blk = static_cast<int64_t>(blockIdx.x) * iters + i;
          col = static_cast<int>(blk % boxes_per_row) * 64;
          row = static_cast<int>(((blk / boxes_per_row) * 128) % rows_total);
        }
        mbar_arrive_expect_tx(&full[s], 16384);
        tma_load_2d(&tm, smem_u32(smem + s * 16384), smem_u32(&full[s]), col, row, 0);
      }
    }
    long long t1 = clock64();
    out[blockIdx.x] = static_cast<unsigned long long>(t1 - t0);
  }
#endif
}

// Streaming pattern study for HBM-bound GEMM operands: each CTA owns bands of
// `box_rows` rows of a [rows x row_len] FP16 tensor (row pitch row_len*2 B) and
// reads them in 128-B-wide boxes with `depth` boxes in flight.
//   order 0: GEMM order -- walk the k (column) boxes of a band, then the next band
//   order 1: contiguous order -- the band's boxes column-major in memory order
//            only when row_len == 64 (one box per row band); else same as 0
__global__ void __launch_bounds__(32, 1) tma_stream_kernel(const __grid_constant__ CUtensorMap tm, int row_len,
                                                            int rows, int box_rows, int depth,
                                                            unsigned long long *out) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw & 1023u)) & 1023u);
  const uint32_t box_bytes = static_cast<uint32_t>(box_rows) * 128u;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + depth * box_bytes);
  if (threadIdx.x == 0) {
    for (int s = 0; s < depth; ++s) mbar_init(&full[s], 1);
    fence_mbarrier_init();
  }
  __syncwarp();
  if (threadIdx.x == 0) {
    const int kboxes = row_len / 64;
    const int bands = rows / box_rows;
    const int my_bands = (bands - static_cast<int>(blockIdx.x) + static_cast<int>(gridDim.x) - 1) / static_cast<int>(gridDim.x);
    const int total = my_bands * kboxes;
    long long t0 = clock64();
    uint32_t phase = 0;
    for (int i = 0; i < total + depth; ++i) {
      const int s = i % depth;
      if (i >= depth) {
        mbar_wait(&full[s], phase);
        if (s == depth - 1) phase ^= 1u;
      }
      if (i < total) {
        const int band = static_cast<int>(blockIdx.x) + (i / kboxes) * static_cast<int>(gridDim.x);
        const int col = (i % kboxes) * 64;
        mbar_arrive_expect_tx(&full[s], box_bytes);
        tma_load_2d(&tm, smem_u32(smem + s * box_bytes), smem_u32(&full[s]), col, band * box_rows, 0);
      }
    }
    long long t1 = clock64();
    out[blockIdx.x] = static_cast<unsigned long long>(t1 - t0);
  }
#endif
}

// The same study with G consecutive k boxes of a band fetched by ONE 3-D TMA
// load (tensor map dims {64, rows, row_len/64}, strides {pitch, 128 B}; box
// {64, box_rows, G}): the shared-memory image is G ordinary SW128 k-block
// tiles back to back, but the TMA engine requests G x 128 contiguous bytes of
// every row at once.
__global__ void __launch_bounds__(32, 1) tma_stream3d_kernel(const __grid_constant__ CUtensorMap tm, int row_len,
                                                              int rows, int box_rows, int g, int depth,
                                                              unsigned long long *out) {
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t *smem = smem_raw + ((1024u - (raw & 1023u)) & 1023u);
  const uint32_t slot_bytes = static_cast<uint32_t>(box_rows) * 128u * static_cast<uint32_t>(g);
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + depth * slot_bytes);
  if (threadIdx.x == 0) {
    for (int s = 0; s < depth; ++s) mbar_init(&full[s], 1);
    fence_mbarrier_init();
  }
  __syncwarp();
  if (threadIdx.x == 0) {
    const int kgroups = row_len / (64 * g);
    const int bands = rows / box_rows;
    const int my_bands = (bands - static_cast<int>(blockIdx.x) + static_cast<int>(gridDim.x) - 1) / static_cast<int>(gridDim.x);
    const int total = my_bands * kgroups;
    long long t0 = clock64();
    uint32_t phase = 0;
    for (int i = 0; i < total + depth; ++i) {
      const int s = i % depth;
      if (i >= depth) {
        mbar_wait(&full[s], phase);
        if (s == depth - 1) phase ^= 1u;
      }
      if (i < total) {
        const int band = static_cast<int>(blockIdx.x) + (i / kgroups) * static_cast<int>(gridDim.x);
        const int kb = (i % kgroups) * g;
        mbar_arrive_expect_tx(&full[s], slot_bytes);
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(smem + s * slot_bytes)),
            "l"(reinterpret_cast<uint64_t>(&tm)), "r"(smem_u32(&full[s])), "r"(0), "r"(band * box_rows), "r"(kb)
            : "memory");
      }
    }
    long long t1 = clock64();
    out[blockIdx.x] = static_cast<unsigned long long>(t1 - t0);
  }
#endif
}

// Plain vectorised global loads over n16 16-byte words (reference read rate):
// grid-stride, 8 independent 16-B loads in flight per thread, xor-reduced.
__global__ void __launch_bounds__(512) ldg_read_kernel(const uint4 *src, int64_t n16, unsigned long long *out) {
  uint32_t acc = 0;
  const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
  int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n16; i += 8 * stride) {
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldcs(src + i + u * stride);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  for (; i < n16; i += stride) {
    const uint4 v = __ldcs(src + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x9e3779b9u) out[0] = acc;  // keeps the loads live
}

}  // namespace mb

namespace {
using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  }
  return fn;
}
}  // namespace

__global__ void stamp_kernel(unsigned long long *dst) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  *dst = t;
}

__global__ void empty_kernel(unsigned long long *dst, int touch_smem) {
  extern __shared__ uint8_t sm[];
  if (touch_smem && threadIdx.x == 0) sm[0] = 1;
  if (dst && threadIdx.x == 0 && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    *dst = t;
  }
}

// Teardown probes (tools/teardown_probe.py): an otherwise empty kernel that
// mode & 1: allocates and frees 512 TMEM columns (cta_group::1, or ::2 when the
//           cluster has 2 CTAs), like the GEMM kernels;
// mode & 2: issues one 4 KB bulk store (shared -> global) per warp and exits after
//           its shared-memory read completed (the global write still in flight),
//           like the GEMM epilogue;
// mode & 4: executes griddepcontrol.launch_dependents early (PDL trigger).
template <int CG>
__global__ void teardown_kernel(int mode, uint8_t *gdst) {
  using namespace hg;
#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ >= 1000)
  extern __shared__ uint8_t sm[];
  __shared__ uint32_t slot;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (mode & 4) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if ((mode & 1) && warp == 1) tmem_alloc<CG>(smem_u32(&slot), 512);
  if (mode & 2) {
    for (int i = threadIdx.x; i < 1024 * (blockDim.x / 32); i += blockDim.x) sm[i] = static_cast<uint8_t>(i);
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();
  tc_fence_after();
  if ((mode & 2) && lane == 0) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    const size_t off = (static_cast<size_t>(blockIdx.x) * (blockDim.x / 32) + warp) * 4096;
    bulk_store_1d(gdst + off, smem_u32(sm) + warp * 4096 % (1024 * (blockDim.x / 32)), 4096);
    bulk_commit_group();
    hg::bulk_wait_group_read<0>();
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();
  if ((mode & 1) && warp == 1) {
    tc_fence_after();
    tmem_dealloc<CG>(slot, 512);
  }
#endif
}

// Placement probe: every CTA of a cluster launch (the GEMM's shape) records %smid.
__global__ void smid_kernel(int *out) {
  extern __shared__ uint8_t sm[];
  if (threadIdx.x == 0) {
    uint32_t id;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(id));
    out[blockIdx.x] = static_cast<int>(id);
    sm[0] = 1;
  }
}

extern "C" {

// out[b] = %smid of CTA b for a grid of `grid` CTAs in clusters of `cluster` with `smem` bytes.
int mb_smid(int grid, int cluster, int smem, int *out, cudaStream_t s) {
  if (cudaFuncSetAttribute(smid_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448) != cudaSuccess)
    return 2;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(128);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeClusterDimension;
  a[0].val.clusterDim.x = cluster;
  a[0].val.clusterDim.y = 1;
  a[0].val.clusterDim.z = 1;
  cfg.attrs = a;
  cfg.numAttrs = cluster > 0 ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, smid_kernel, out) == cudaSuccess ? 0 : 1;
}

int mb_teardown(int grid, int block, int smem, int cluster, int mode, int pdl, void *gdst, cudaStream_t s) {
  static int attr = 0;
  if (!attr) {
    if (cudaFuncSetAttribute(teardown_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) !=
            cudaSuccess ||
        cudaFuncSetAttribute(teardown_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) !=
            cudaSuccess)
      return 2;
    attr = 1;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute a[2];
  int na = 0;
  if (cluster > 0) {
    a[na].id = cudaLaunchAttributeClusterDimension;
    a[na].val.clusterDim.x = cluster;
    a[na].val.clusterDim.y = 1;
    a[na].val.clusterDim.z = 1;
    ++na;
  }
  if (pdl) {
    a[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    a[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  cfg.attrs = a;
  cfg.numAttrs = na;
  cudaError_t e = cluster == 2 ? cudaLaunchKernelEx(&cfg, teardown_kernel<2>, mode, static_cast<uint8_t *>(gdst))
                               : cudaLaunchKernelEx(&cfg, teardown_kernel<1>, mode, static_cast<uint8_t *>(gdst));
  return e == cudaSuccess ? 0 : 1;
}

// Empty kernel with the tile kernel's launch shape (grid, block, dynamic smem,
// cluster size): the fixed cost of such a launch, nothing else.
int mb_empty(int grid, int block, int smem, int cluster, unsigned long long *dst, cudaStream_t s) {
  static int attr = 0;
  if (!attr) {
    if (cudaFuncSetAttribute(empty_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448) != cudaSuccess)
      return 2;
    attr = 1;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeClusterDimension;
  a[0].val.clusterDim.x = cluster;
  a[0].val.clusterDim.y = 1;
  a[0].val.clusterDim.z = 1;
  cfg.attrs = a;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, empty_kernel, dst, smem > 0 ? 1 : 0) == cudaSuccess ? 0 : 1;
}

// cudaOccupancyMaxActiveClusters for a kernel of this launch shape (cluster size,
// dynamic smem, block): how many clusters of that size the GPU holds at once.
int mb_max_clusters(int cluster, int smem, int block) {
  if (cudaFuncSetAttribute(empty_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448) != cudaSuccess)
    return -2;
  if (cluster > 8 && cudaFuncSetAttribute(empty_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess)
    return -3;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(cluster * 64);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeClusterDimension;
  a[0].val.clusterDim.x = cluster;
  a[0].val.clusterDim.y = 1;
  a[0].val.clusterDim.z = 1;
  cfg.attrs = a;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, empty_kernel, &cfg) != cudaSuccess) return -1;
  return n;
}

// One-thread kernel writing %globaltimer to *dst (timeline probes around a launch).
int mb_stamp(unsigned long long *dst, cudaStream_t s) {
  stamp_kernel<<<1, 32, 0, s>>>(dst);
  return cudaPeekAtLastError() == cudaSuccess ? 0 : 1;
}

// cycles[i] for CTA (or CTA pair) i; returns 0 on success.
int mb_mma_rate(int cta_group, int n, int iters, int grid, int latency_mode, unsigned long long *cycles_dev) {
  const int smem = 16384 + 256 * 128 + 1024 + 1024;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(128);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = cta_group;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
#define MB_CASE(CG, NN)                                                                               \
  if (cta_group == CG && n == NN) {                                                                   \
    auto k = mb::mma_rate_kernel<CG, NN>;                                                             \
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);                       \
    return cudaLaunchKernelEx(&cfg, k, iters, cycles_dev, latency_mode) == cudaSuccess ? 0 : 1;       \
  }
  MB_CASE(1, 64)
  MB_CASE(1, 128)
  MB_CASE(1, 256)
  MB_CASE(2, 64)
  MB_CASE(2, 128)
  MB_CASE(2, 256)
#undef MB_CASE
  return 2;
}

int mb_tmem_ld(int iters, int warps, int unroll, int grid, unsigned long long *cycles_dev) {
  mb::tmem_ld_kernel<<<grid, 256>>>(iters, warps, unroll, cycles_dev);
  return cudaPeekAtLastError() == cudaSuccess ? 0 : 1;
}

// tensor: rows x 512 FP16 row-major device buffer (rows multiple of 128)
int mb_tma_load(const void *tensor, int rows, int iters, int grid, int streaming, unsigned long long *cycles_dev) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return 3;
  CUtensorMap tm;
  cuuint64_t dims[2] = {512, static_cast<cuuint64_t>(rows)};
  cuuint64_t strides[1] = {512 * 2};
  cuuint32_t box[2] = {64, 128};
  cuuint32_t estr[2] = {1, 1};
  if (fn(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void *>(tensor), dims, strides, box, estr,
         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return 4;
  const int smem = 8 * 16384 + 1024 + 1024;
  cudaFuncSetAttribute(mb::tma_load_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  mb::tma_load_kernel<<<grid, 32, smem>>>(tm, iters, rows, streaming, cycles_dev);
  return cudaPeekAtLastError() == cudaSuccess ? 0 : 1;
}

}  // extern "C"

// Streaming pattern study (see tma_stream_kernel); returns 0 on success.
extern "C" int mb_tma_stream(const void *tensor, int row_len, int rows, int box_rows, int depth, int grid,
                             unsigned long long *cycles_dev) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return 3;
  CUtensorMap tm;
  cuuint64_t dims[2] = {static_cast<cuuint64_t>(row_len), static_cast<cuuint64_t>(rows)};
  cuuint64_t strides[1] = {static_cast<cuuint64_t>(row_len) * 2};
  cuuint32_t box[2] = {64, static_cast<cuuint32_t>(box_rows)};
  cuuint32_t estr[2] = {1, 1};
  if (fn(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void *>(tensor), dims, strides, box, estr,
         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return 2;
  const int smem = depth * box_rows * 128 + 1024 + 1024;
  if (cudaFuncSetAttribute(mb::tma_stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
    return 1;
  mb::tma_stream_kernel<<<grid, 32, smem>>>(tm, row_len, rows, box_rows, depth, cycles_dev);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}

extern "C" int mb_tma_stream3d(const void *tensor, int row_len, int rows, int box_rows, int g, int depth, int grid,
                               unsigned long long *cycles_dev) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return 3;
  CUtensorMap tm;
  cuuint64_t dims[3] = {64, static_cast<cuuint64_t>(rows), static_cast<cuuint64_t>(row_len / 64)};
  cuuint64_t strides[2] = {static_cast<cuuint64_t>(row_len) * 2, 128};
  cuuint32_t box[3] = {64, static_cast<cuuint32_t>(box_rows), static_cast<cuuint32_t>(g)};
  cuuint32_t estr[3] = {1, 1, 1};
  if (fn(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, const_cast<void *>(tensor), dims, strides, box, estr,
         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return 2;
  const int smem = depth * box_rows * 128 * g + 1024 + 1024;
  if (smem > 227 * 1024) return 4;
  if (cudaFuncSetAttribute(mb::tma_stream3d_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
    return 1;
  mb::tma_stream3d_kernel<<<grid, 32, smem>>>(tm, row_len, rows, box_rows, g, depth, cycles_dev);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}

extern "C" int mb_ldg_read(const void *src, long long bytes, int grid, int block, unsigned long long *out_dev) {
  mb::ldg_read_kernel<<<grid, block>>>(static_cast<const uint4 *>(src), bytes / 16, out_dev);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
