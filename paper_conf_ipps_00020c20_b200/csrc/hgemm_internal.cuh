// Host-side internals shared by the translation units of libhgemm.so:
// hgemm_api.cu (the C ABI, validation, kernel choice, tensor maps) and the
// hgemm_inst_*.cu files, each of which instantiates and launches one family of
// kernels (so that the library builds in parallel, one nvcc per family).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdint>
#include <mutex>

#include "../../include/hgemm.h"
#include "hgemm_splitk.cuh"
#include "hgemm_tc.cuh"

namespace hgi {

constexpr int kMaxDevices = 64;

struct DeviceInfo {
  bool init = false;
  bool ok = false;
  int num_sms = 0;
};

extern std::atomic<int64_t> g_launches;  // kernel launches enqueued by this process
extern const bool g_pdl;                  // programmatic dependent launch (HGEMM_PDL=0 disables it)
extern thread_local bool t_half_used;     // the last tile launch of this thread used the half-tile tail

// Stream-K plan (hgemm_api.cu): number of data-parallel tiles, or -1 for "no stream-K".
int sk_plan(int64_t tiles, int64_t units, int64_t nkb, int mode);
// Library-owned stream-K partial slots and flags for (device, stream) (hgemm_api.cu);
// flags + kWsyncOffset is the wave-barrier counter.
bool sk_workspace(int dev, cudaStream_t s, int num_sms, float **ws, int **flags);
extern const int kWsyncOffset;
extern const int g_env_wsync;  // HGEMM_WSYNC: 1 = wave barrier for tile kernels with >= 8 whole waves
extern const int g_env_wsync_minw;  // HGEMM_WSYNC_MINW: minimum whole waves for the wave barrier (default 8)
extern const int g_env_wsync_k;  // HGEMM_WSYNC_K: k-block interval of extra barriers inside tiles (0 = none, -1 = auto)

// One launch of a persistent tile kernel.
struct TcLaunch {
  const CUtensorMap *ta, *tb, *td;
  const hg::TcParams *p;
  int dev;
  const DeviceInfo *di;
  int max_ctas;   // cap on CTAs (0 = all SMs)
  int sk_mode;    // hgemm_config_t::stream_k | hgemm_config_t::half_tail << 4
  bool *sk_used;  // out: stream-K was used
  cudaStream_t stream;
};

// Per-family dispatchers (layout flags -> template instantiation), one per TU.
//   acc16: FP16 accumulation (c_format = F16), FP16 output only, no all-gather / multicast.
hgemm_status_t dispatch_tc512(int mc, bool ag, bool acc16, bool a_mn, bool b_mn, bool f32, const TcLaunch &L);
hgemm_status_t dispatch_tc256x2(int mc, bool ag, bool acc16, bool a_mn, bool b_mn, bool f32, const TcLaunch &L,
                                bool direct = false);
hgemm_status_t dispatch_tc1(int bn, bool a_mn, bool b_mn, bool f32, const TcLaunch &L);
// 256-wide CTA-pair tiles with k-group stages (KG = 2): TN layout,
// K % 128 == 0, whole tiles; tensor maps are the 3-D k-group views (box {64, rows, 2})
hgemm_status_t dispatch_tc256_kg2(int cg, bool f32, const TcLaunch &L, int mc = 1);
hgemm_status_t dispatch_splitk64(int spl, bool a_mn, bool b_mn, bool f32, const CUtensorMap &ta,
                                 const CUtensorMap &tb, const hg::TcParams &p, int dev, cudaStream_t s,
                                 bool hm = false);
hgemm_status_t dispatch_splitk128(int spl, bool a_mn, bool b_mn, bool f32, const CUtensorMap &ta,
                                  const CUtensorMap &tb, const hg::TcParams &p, int dev, cudaStream_t s);

// ----------------------------------------------------------------- tile kernel launch
// Per-instantiation, per-device one-time setup (dynamic smem attribute, resident
// cluster count), thread-safe: concurrent first calls all see the finished setup.
// One function-local static per launch_* instantiation.
struct KernInit {
  std::once_flag once[kMaxDevices];
  cudaError_t err[kMaxDevices] = {};
  int max_clusters[kMaxDevices] = {};
};

template <int BN, int CG, bool A_MN, bool B_MN, bool OUT_F32, int MC, bool AG, bool ACC16, bool DIRECT = false,
          int KG = 1>
hgemm_status_t launch_tc(const TcLaunch &L) {
  using S = hg::TcShape<BN, CG, OUT_F32, DIRECT, KG>;
  constexpr int THREADS = S::THREADS + (AG ? 32 : 0);  // + the all-gather copy warp
  const int dev = L.dev;
  const DeviceInfo &di = *L.di;
  const hg::TcParams &p0 = *L.p;
  const int ht_mode = L.sk_mode >> 4;  // hgemm_config_t::half_tail, packed above the stream-K mode
  const int sk_mode = L.sk_mode & 15;
  auto kern = hg::hgemm_tc_kernel<BN, CG, A_MN, B_MN, OUT_F32, MC, AG, ACC16, DIRECT, KG>;
  static KernInit init;
  std::call_once(init.once[dev], [&] {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, S::SMEM_BYTES);
    int n = di.num_sms;
    if (e == cudaSuccess && CG == 2) {
      cudaLaunchConfig_t qc = {};
      qc.gridDim = dim3(CG * MC * (di.num_sms / (CG * MC)));
      qc.blockDim = dim3(THREADS);
      qc.dynamicSmemBytes = S::SMEM_BYTES;
      cudaLaunchAttribute qa[1];
      qa[0].id = cudaLaunchAttributeClusterDimension;
      qa[0].val.clusterDim.x = CG * MC;
      qa[0].val.clusterDim.y = 1;
      qa[0].val.clusterDim.z = 1;
      qc.attrs = qa;
      qc.numAttrs = 1;
      n = 0;
      if (cudaOccupancyMaxActiveClusters(&n, kern, &qc) != cudaSuccess || n <= 0) {
        (void)cudaGetLastError();
        n = di.num_sms / (CG * MC);
      }
    }
    init.max_clusters[dev] = std::max(1, n);
    init.err[dev] = e;
  });
  if (init.err[dev] != cudaSuccess) return HGEMM_ERR_CUDA;
  const int tiles = p0.num_m_tiles * p0.num_n_tiles;
  int units = init.max_clusters[dev];
  if (L.max_ctas > 0) units = std::max(1, std::min(units, L.max_ctas / (CG * MC)));
  int clusters = std::min(tiles, units);
  hg::TcParams p = p0;
  p.dp_tiles = tiles;
  p.sk_u0 = p.sk_units = 0;
  p.sk_ws = nullptr;
  p.sk_flags = nullptr;
  p.n_half = 0;
  *L.sk_used = false;
  // half-tile tail (512-wide tiles): a last wave of r <= units/2 tiles runs as 2r
  // 256-wide items, i.e. in about half the time
  bool half_tail = false;
  if (BN == 512 && CG == 2 && MC == 1 && !AG && ht_mode != 1 && sk_mode != 2) {
    const int r = tiles % units;
    if (r > 0 && 2 * r <= units && (ht_mode == 2 || tiles / units >= 4)) {
      p.n_half = r;
      p.dp_tiles = tiles + r;
      clusters = std::min(tiles + r, units);
      half_tail = true;
    }
  }
  t_half_used = half_tail;
  if (MC == 1 && !AG && !ACC16 && !half_tail) {
    // k-group stages (KG = 2): stream-K units of KG k-blocks, so every item starts and ends on
    // a stage boundary
    const int nku = p.num_k_blocks / KG;
    const int dp = sk_plan(tiles, units, nku, sk_mode);
    float *ws = nullptr;
    int *flags = nullptr;
    if (dp >= 0 && units * CG * MC <= di.num_sms && sk_workspace(dev, L.stream, di.num_sms, &ws, &flags)) {
      p.dp_tiles = dp;
      p.sk_kgu = KG;
      p.sk_u0 = static_cast<int64_t>(dp) * nku;
      p.sk_units = static_cast<int64_t>(tiles - dp) * nku;
      p.sk_ws = ws;
      p.sk_flags = flags;
      clusters = units;
      *L.sk_used = true;
    }
  }
  // Wave barrier: with >= 8 whole waves of whole tiles and K >= 8192, the
  // producers of all CTAs meet before each wave, so the tiles that share Ak / Bk panels
  // stream their k-blocks together instead of drifting apart over the waves (at 32768^3 the
  // DRAM reads fall from 165 to 52 GB per launch).  Needs every cluster resident at once, as
  // the grid is sized for (the stream-K fix-up relies on the same).  HGEMM_WSYNC=0 disables it.
  p.wsync = nullptr;
  p.wsync_items = 0;
  p.wsync_kint = 0;
  // (the fused all-gather kernel too: its copy warps never wait on a producer, so a producer
  // held at the meeting cannot block the copies another producer is waiting for)
  if (g_env_wsync && MC == 1 && !*L.sk_used && clusters == units) {
    const int whole_waves = (tiles - p.n_half) / units;
    float *ws = nullptr;
    int *flags = nullptr;
    // long tiles only (K >= 8192): with short k loops the panels stay in L2 anyway and the
    // per-wave meeting costs more than it saves (BERT-FFN1 16384 x 4096 x 1024: 129 -> 151 us)
    if (whole_waves >= g_env_wsync_minw && p.num_k_blocks >= 128 && units * CG <= di.num_sms &&
        sk_workspace(dev, L.stream, di.num_sms, &ws, &flags) &&
        cudaMemsetAsync(flags + kWsyncOffset, 0, sizeof(int), L.stream) == cudaSuccess) {
      p.wsync = flags + kWsyncOffset;
      p.wsync_items = whole_waves;
      // inside long tiles also every 64 k-blocks: at K >= 16384 the L2 read sectors fell by 16%
      // and the sustained rate rose 1.5-3% (profiles/r02/wave_barrier_k_interval.log)
      p.wsync_kint = g_env_wsync_k >= 0 ? g_env_wsync_k : (p.num_k_blocks >= 256 ? 64 : 0);
    }
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(clusters * CG * MC);
  cfg.blockDim = dim3(THREADS);
  cfg.dynamicSmemBytes = S::SMEM_BYTES;
  cfg.stream = L.stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG * MC;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  // programmatic dependent launch: the prologue overlaps the previous kernel's tail
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  if (CG * MC == 1 && (p.exp_flags & 16)) {  // experiment: plain (non-cluster) launch for 1-CTA "clusters"
    cfg.attrs = attr + 1;
    cfg.numAttrs = 1;
  }
  if (cudaLaunchKernelEx(&cfg, kern, *L.ta, *L.tb, *L.td, p) != cudaSuccess) return HGEMM_ERR_CUDA;
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return HGEMM_SUCCESS;
}

// All eight (op(B) MN-major, op(A) MN-major, FP32 out) combinations of one tile shape.
template <int BN, int CG, int MC, bool DIRECT = false>
hgemm_status_t dispatch_tc_layout(bool a_mn, bool b_mn, bool f32, const TcLaunch &L) {
#define HG_CASE(AM, BM_, F) \
  if (a_mn == AM && b_mn == BM_ && f32 == F) return launch_tc<BN, CG, AM, BM_, F, MC, false, false, DIRECT>(L);
  HG_CASE(false, false, false)
  HG_CASE(false, false, true)
  HG_CASE(false, true, false)
  HG_CASE(false, true, true)
  HG_CASE(true, false, false)
  HG_CASE(true, false, true)
  HG_CASE(true, true, false)
  HG_CASE(true, true, true)
#undef HG_CASE
  return HGEMM_ERR_INVALID_VALUE;
}

// FP16-accumulate kernels (FP16 output): the four layouts of one CTA-pair tile shape.
template <int BN>
hgemm_status_t dispatch_tc_acc16(bool a_mn, bool b_mn, const TcLaunch &L) {
  if (!a_mn && !b_mn) return launch_tc<BN, 2, false, false, false, 1, false, true>(L);
  if (!a_mn && b_mn) return launch_tc<BN, 2, false, true, false, 1, false, true>(L);
  if (a_mn && !b_mn) return launch_tc<BN, 2, true, false, false, 1, false, true>(L);
  return launch_tc<BN, 2, true, true, false, 1, false, true>(L);
}

// Fused all-gather kernels: CTA pairs, op(A) K-major (transA = 'T').
template <int BN>
hgemm_status_t dispatch_tc_ag(bool a_mn, bool f32, const TcLaunch &L) {
  TcLaunch l2 = L;
  l2.sk_mode = 1;  // stream-K off: its work items do not follow the chunk order
  if (!a_mn && !f32) return launch_tc<BN, 2, false, false, false, 1, true, false>(l2);
  if (!a_mn && f32) return launch_tc<BN, 2, false, false, true, 1, true, false>(l2);
  if (a_mn && !f32) return launch_tc<BN, 2, true, false, false, 1, true, false>(l2);
  return launch_tc<BN, 2, true, false, true, 1, true, false>(l2);
}

// ----------------------------------------------------------------- split-K launch
template <int BN, int SPL, bool A_MN, bool B_MN, bool OUT_F32, bool HM = false>
hgemm_status_t launch_splitk(const CUtensorMap &ta, const CUtensorMap &tb, const hg::TcParams &p, int dev,
                             cudaStream_t stream) {
  using SH = hg::SkShape<BN, SPL, HM>;
  auto kern = hg::hgemm_splitk_kernel<BN, SPL, A_MN, B_MN, OUT_F32, HM>;
  static KernInit init;
  std::call_once(init.once[dev], [&] {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SH::SMEM_BYTES);
    if (e == cudaSuccess && SPL > 8) e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    init.err[dev] = e;
  });
  if (init.err[dev] != cudaSuccess) return HGEMM_ERR_CUDA;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(static_cast<unsigned>(p.num_m_tiles * p.num_n_tiles * SPL));
  cfg.blockDim = dim3(192);
  cfg.dynamicSmemBytes = SH::SMEM_BYTES;
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = SPL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  if (cudaLaunchKernelEx(&cfg, kern, ta, tb, p) != cudaSuccess) return HGEMM_ERR_CUDA;
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return HGEMM_SUCCESS;
}

template <int BN, int SPL, bool HM = false>
hgemm_status_t dispatch_splitk_layout(bool a_mn, bool b_mn, bool f32, const CUtensorMap &ta, const CUtensorMap &tb,
                                      const hg::TcParams &p, int dev, cudaStream_t s) {
#define HG_SK(AM, BM_, F) \
  if (a_mn == AM && b_mn == BM_ && f32 == F) return launch_splitk<BN, SPL, AM, BM_, F, HM>(ta, tb, p, dev, s);
  HG_SK(false, false, false)
  HG_SK(false, false, true)
  HG_SK(false, true, false)
  HG_SK(false, true, true)
  HG_SK(true, false, false)
  HG_SK(true, false, true)
  HG_SK(true, true, false)
  HG_SK(true, true, true)
#undef HG_SK
  return HGEMM_ERR_INVALID_VALUE;
}

}  // namespace hgi
