// Host runtime behind the C ABI of include/hgemm.h: argument validation,
// BLAS quick returns, kernel selection, TMA tensor-map encoding and launch.
//
// Mapping of the column-major ABI onto the kernel (hgemm_tc.cuh):
//   D = C^T (row-major, ldd = ldc), M = n, N = m,
//   Ak = op(B)^T  (n x k): transB 'N' -> K-major rows of B; 'T' -> MN-major
//   Bk = op(A)    (m x k): transA 'T' -> K-major rows of A; 'N' -> MN-major
// The paper's benchmark layout (A row-major, B column-major)
// is transA = 'T', transB = 'N': both operands K-major.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "../../include/hgemm.h"
#include "hgemm_internal.cuh"
#include "hgemm_simt.cuh"
#include "hgemm_stream.cuh"


// ----------------------------------------------------------------- shared state (hgemm_internal.cuh)
namespace hgi {
std::atomic<int64_t> g_launches{0};
extern const bool g_pdl = [] {
  const char *e = std::getenv("HGEMM_PDL");
  return !(e && e[0] == '0');
}();
thread_local bool t_half_used = false;
}  // namespace hgi

namespace {

using hg::TcParams;
using hgi::DeviceInfo;
using hgi::g_launches;
using hgi::g_pdl;
using hgi::kMaxDevices;
using hgi::t_half_used;

// ----------------------------------------------------------------- device info
DeviceInfo g_dev[kMaxDevices];
std::mutex g_mu;

hgemm_config_t g_cfg = {HGEMM_KERNEL_AUTO, 0, 0, 0, 0, 0, 0, 0};
hgemm_config_t g_last = {HGEMM_KERNEL_AUTO, 0, 0, 0, 0, 0, 0, 0};
std::atomic<unsigned long long *> g_probe{nullptr};
// experiment knobs, read once at load time (never per call)
int env_int(const char *name, int dflt) {
  const char *e = std::getenv(name);
  return e ? std::atoi(e) : dflt;
}
const int g_env_stream_rot = env_int("HGEMM_STREAM_ROT", 1);  // streaming kernel k rotation
const int g_env_stream_stages = env_int("HGEMM_STREAM_STAGES", 0);  // experiments: cap on the streaming ring depth
const int g_env_stream_g = env_int("HGEMM_STREAM_G", -1);  // streaming kernel k-blocks per stage (3-D Bk map); -1: auto
const int g_env_stream_mmax = env_int("HGEMM_STREAM_MMAX", 128);  // largest M (= n) the streaming kernel is chosen for
const int g_env_sk_b3d = env_int("HGEMM_SK_B3D", 1);          // split-K: op(A) through the 3-D k-group view
const int g_env_sk_kg = env_int("HGEMM_SK_KG", 2);            // split-K kernel k-blocks per stage (1 or 2)
const int g_env_stream_pre = env_int("HGEMM_STREAM_PRE", 0);    // streaming kernel stage loads before the CTA barrier (0: all)
const int g_env_mc = env_int("HGEMM_MC", 1);                  // 2: multicast pair kernel (-DHGEMM_ENABLE_MC)
const int g_env_group_n = env_int("HGEMM_GROUP_N", 0);        // > 0: raster groups along N
const int g_env_l2_hint = env_int("HGEMM_L2_HINT", 0);        // TMA L2 cache hints
const int g_env_sk_hm = env_int("HGEMM_SK_HM", 0);            // split-K 64-wide: 64-row tiles (experiments)
const int g_env_exp = env_int("HGEMM_EXP", 0);                // TcParams::exp_flags
const bool g_env_flex = env_int("HGEMM_FLEX", 0) != 0;        // flexible tile widths in the automatic choice
const int g_env_stream_a3d = env_int("HGEMM_STREAM_A3D", 1);  // streaming kernel: Ak through the 3-D k-group view
const int g_env_tc_kg = env_int("HGEMM_TC_KG", 2);            // 256-wide pair / 128 x 128 tiles: k-blocks per ring stage (1 or 2)
const int g_env_tc_kg_sk = env_int("HGEMM_TC_KG_SK", 1);      // k-group stages also with stream-K (units of 2 k-blocks)
const int g_env_tc1_kg = env_int("HGEMM_TC1_KG", 1);          // k-group stages for 1-SM 128 x 128 tiles too
const int g_env_direct = env_int("HGEMM_EPI_DIRECT", 0);      // 256-wide pair tiles: direct-store epilogue, 7 stages

bool device_info(int dev, DeviceInfo &out) {
  if (dev < 0 || dev >= kMaxDevices) return false;
  std::lock_guard<std::mutex> lk(g_mu);
  DeviceInfo &d = g_dev[dev];
  if (!d.init) {
    int major = 0, minor = 0, sms = 0;
    if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
      return false;
    }
    d.ok = (major == 10 && minor == 0);
    d.num_sms = sms;
    d.init = true;
  }
  out = d;
  return true;
}

// ----------------------------------------------------------------- tensor maps
using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess) {
      fn = reinterpret_cast<EncodeTiledFn>(p);
    }
  });
  return fn;
}

// 2-D tensor with 128-B swizzled boxes: `inner` contiguous elements per line,
// `outer` lines `ld` elements apart.  FP16 operands (loads) or the FP16/FP32
// output D (epilogue stores).  Encoded maps are cached (keyed by every encode
// argument): repeated calls on the same buffers skip cuTensorMapEncodeTiled.
// A cached map is a plain value copied into the launch parameters; nothing is
// dereferenced on the host.
struct MapKey {
  const void *base;
  uint64_t inner, outer;
  int64_t ld;
  uint32_t box_inner, box_outer;
  int f32;
  int g3d;  // 0: the 2-D map; G > 0: the 3-D k-block-grouped view with G k-blocks per box
  bool operator==(const MapKey &o) const {
    return base == o.base && inner == o.inner && outer == o.outer && ld == o.ld && box_inner == o.box_inner &&
           box_outer == o.box_outer && f32 == o.f32 && g3d == o.g3d;
  }
};
constexpr int kMapCache = 32;
struct MapCache {
  MapKey key[kMapCache];
  CUtensorMap map[kMapCache];
  bool valid[kMapCache] = {};
  int next = 0;
  std::mutex mu;
};
MapCache g_maps;

bool make_map(CUtensorMap *map, const void *base, uint64_t inner, uint64_t outer, int64_t ld, uint32_t box_inner,
              uint32_t box_outer, bool f32 = false) {
  const MapKey key = {base, inner, outer, ld, box_inner, box_outer, f32 ? 1 : 0, 0};
  {
    std::lock_guard<std::mutex> lk(g_maps.mu);
    for (int i = 0; i < kMapCache; ++i)
      if (g_maps.valid[i] && g_maps.key[i] == key) {
        *map = g_maps.map[i];
        return true;
      }
  }
  EncodeTiledFn fn = encode_fn();
  if (!fn) return false;
  const int esz = f32 ? 4 : 2;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {static_cast<cuuint64_t>(ld) * esz};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  static const CUtensorMapL2promotion promo = [] {  // experiments: HGEMM_L2_PROMO = 0/64/128/256
    const char *e = std::getenv("HGEMM_L2_PROMO");
    const int v = e ? std::atoi(e) : 256;
    return v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE : v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
           : v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  }();
  CUresult r = fn(map, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2,
                  const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_128B, promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  std::lock_guard<std::mutex> lk(g_maps.mu);
  const int slot = g_maps.next;
  g_maps.next = (g_maps.next + 1) % kMapCache;
  g_maps.key[slot] = key;
  g_maps.map[slot] = *map;
  g_maps.valid[slot] = true;
  return true;
}

// 3-D k-block-grouped view of a K-major FP16 operand (`inner` = K, a multiple
// of 64; `outer` rows `ld` elements apart): dims {64, outer, K/64}, strides
// {ld, 128 B}, box {64, box_outer, g}.  One load brings g consecutive k-blocks
// of box_outer rows as g ordinary SW128 k-block tiles back to back.
bool make_map_3d(CUtensorMap *map, const void *base, uint64_t inner, uint64_t outer, int64_t ld, uint32_t box_outer,
                 uint32_t g) {
  const MapKey key = {base, inner, outer, ld, 64, box_outer, 0, static_cast<int>(g)};
  {
    std::lock_guard<std::mutex> lk(g_maps.mu);
    for (int i = 0; i < kMapCache; ++i)
      if (g_maps.valid[i] && g_maps.key[i] == key) {
        *map = g_maps.map[i];
        return true;
      }
  }
  EncodeTiledFn fn = encode_fn();
  if (!fn || inner % 64 != 0) return false;
  cuuint64_t dims[3] = {64, outer, inner / 64};
  cuuint64_t strides[2] = {static_cast<cuuint64_t>(ld) * 2, 128};
  cuuint32_t box[3] = {64, box_outer, g};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, const_cast<void *>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  std::lock_guard<std::mutex> lk(g_maps.mu);
  const int slot = g_maps.next;
  g_maps.next = (g_maps.next + 1) % kMapCache;
  g_maps.key[slot] = key;
  g_maps.map[slot] = *map;
  g_maps.valid[slot] = true;
  return true;
}

}  // namespace

namespace hgi {
// ----------------------------------------------------------------- stream-K
// Stream-K plan for `tiles` tiles of `nkb` k-blocks on `units` persistent
// clusters: whole waves minus one run data-parallel, the rest is split into
// one contiguous k range per cluster.  mode: 0 auto, 1 never, 2 always.
// Returns the number of data-parallel tiles, or -1 for "no stream-K".
// Every cluster range must hold >= 2 k-blocks (each partial slot is then
// written at most once per launch).
// Cost of stream-K in waves, measured (tools/tile_choice.py): the
// 256-wide tiles are L2-throughput bound, so spreading the same L2 traffic over
// more SMs gains nothing by itself; the FP32 fixup traffic and the lost
// lockstep between clusters sharing panels cost about a third of a wave.  Stream-K
// pays off only when the last data-parallel wave is nearly empty.
double sk_overhead_waves(int64_t nkb) { return 0.35 + 4.0 / static_cast<double>(nkb); }
int sk_plan(int64_t tiles, int64_t units, int64_t nkb, int mode) {
  if (mode == 1 || units <= 1 || tiles % units == 0 || nkb < 2) return -1;
  const int64_t dp = tiles > units ? (tiles / units - 1) * units : 0;
  if ((tiles - dp) * nkb < 2 * units) return -1;
  if (mode == 0) {
    const double waves_dp = static_cast<double>((tiles + units - 1) / units);
    const double waves_sk = static_cast<double>(tiles) / units + sk_overhead_waves(nkb);
    if (nkb < 8 || waves_sk >= waves_dp) return -1;
  }
  return static_cast<int>(dp);
}

// Library-owned FP32 partial slots + flags, one set per (device, stream):
// room for one 128 x 512 FP32 slot and one flag per SM.  Flags are zero
// between launches (every consumer resets the flag it waited for).
extern const int kWsyncOffset = 1024;  // ints: past the per-SM flags, on its own 128-B line
extern const int g_env_wsync = [] {  // wave barrier: on unless HGEMM_WSYNC=0
  const char *e = std::getenv("HGEMM_WSYNC");
  return e ? std::atoi(e) : 1;
}();
extern const int g_env_wsync_k = [] {  // extra barriers every HGEMM_WSYNC_K k-blocks (-1 = automatic)
  const char *e = std::getenv("HGEMM_WSYNC_K");
  return e ? std::max(0, std::atoi(e)) : -1;
}();
extern const int g_env_wsync_minw = [] {  // wave barrier: minimum whole waves (experiments; default 8)
  const char *e = std::getenv("HGEMM_WSYNC_MINW");
  return e ? std::max(1, std::atoi(e)) : 8;
}();
struct SkWorkspace {
  int dev;
  cudaStream_t stream;
  float *ws;
  int *flags;
};
std::mutex g_skws_mu;
SkWorkspace g_skws[256];
int g_skws_n = 0;

bool sk_workspace(int dev, cudaStream_t s, int num_sms, float **ws, int **flags) {
  std::lock_guard<std::mutex> lk(g_skws_mu);
  for (int i = 0; i < g_skws_n; ++i)
    if (g_skws[i].dev == dev && g_skws[i].stream == s) {
      *ws = g_skws[i].ws;
      *flags = g_skws[i].flags;
      return true;
    }
  if (g_skws_n == 256) return false;
  cudaStreamCaptureStatus cs;
  if (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) return false;
  float *w = nullptr;
  int *f = nullptr;
  if (cudaMalloc(&w, static_cast<size_t>(num_sms) * 128 * 512 * sizeof(float)) != cudaSuccess) return false;
  // flags: one per SM, then (at +kWsyncOffset ints) the wave-barrier counter
  if (cudaMalloc(&f, static_cast<size_t>(kWsyncOffset + 32) * sizeof(int)) != cudaSuccess ||
      cudaMemsetAsync(f, 0, static_cast<size_t>(kWsyncOffset + 32) * sizeof(int), s) != cudaSuccess) {
    cudaFree(w);
    if (f) cudaFree(f);
    return false;
  }
  g_skws[g_skws_n++] = {dev, s, w, f};
  *ws = w;
  *flags = f;
  return true;
}

}  // namespace hgi

namespace {
using hgi::sk_plan;
using hgi::sk_overhead_waves;

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Split-K choice for under-filled shapes: returns false if the tile grid
// already fills the GPU.  Cluster sizes of 4 and 8 leave some SMs of a GPC
// unused (148 SMs do not split into 4-CTA clusters evenly), so the
// capacity per split count is taken conservatively.
bool choose_splitk(int64_t M, int64_t N, int64_t K, int num_sms, int &bn, int &spl, bool &hm) {
  const int64_t nkb = cdiv(K, 64);
  hm = false;
  // Small problems (K <= 1024): 128 x 64 tiles split 4 (or 2) ways whenever that is still one
  // wave -- the loads of a launch-bound GEMM spread over more SMs.  Measured (ncu, cold;
  // profiles/r02/small_split_choice.log): 256^3 NN FP32 8.6 -> 7.5 us, 384^3 9.0 -> 6.7,
  // 512^3 8.6 -> 7.0, 512^3 NN FP32 12.5 -> 7.9, 768^3 9.5 -> 7.8 (the 64-wide split 2).
  if (N > 64 && nkb <= 16) {
    const int64_t t64 = cdiv(M, 128) * cdiv(N, 64);
    if (t64 * 2 <= num_sms) {
      bn = 64;
      spl = (t64 * 4 <= num_sms && nkb >= 4) ? 4 : 2;
      // tiny problems: 64-row tiles (HM) while even those, split 4 ways, fill at most half the
      // SMs -- 256^3 NN FP32 7.4 -> 6.4 us (profiles/r02/splitk_hm_ab.log)
      hm = spl == 4 && cdiv(M, 64) * cdiv(N, 64) * 4 <= num_sms / 2;
      if (nkb >= spl) return true;
    }
  }
  bn = N <= 64 ? 64 : 128;
  const int64_t tiles = cdiv(M, 128) * cdiv(N, bn);
  if (tiles * 2 > num_sms) return false;  // at least half the SMs already busy without splitting
  spl = 0;
  const int cands[3] = {8, 4, 2};
  for (int s : cands) {
    const int64_t cap = s == 2 ? num_sms : (num_sms * 7) / 8;
    if (tiles * s <= cap && nkb >= 4 * s) { spl = s; break; }
  }
  return spl != 0;
}
// ----------------------------------------------------------------- HBM-streaming launch
template <int MT, bool F32>
hgemm_status_t launch_stream(const CUtensorMap &ta, const CUtensorMap &tb, const hg::StreamParams &p, int grid,
                             int dev, cudaStream_t stream) {
  auto kern = hg::hgemm_stream_kernel<MT, F32>;
  static hgi::KernInit init;
  std::call_once(init.once[dev], [&] {
    init.err[dev] = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, hg::kStreamSmemBytes);
  });
  if (init.err[dev] != cudaSuccess) return HGEMM_ERR_CUDA;
  const uint32_t pad = p.a_bytes == 8192u ? 8192u : 0u;  // hgemm_stream.cuh: 64-row Ak boxes
  const uint32_t smem = p.stages * p.stage_bytes + pad + 1024u /*align*/ + 512u /*barriers*/;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(static_cast<unsigned>(grid));
  cfg.blockDim = dim3(192);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = g_pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  if (cudaLaunchKernelEx(&cfg, kern, ta, tb, p) != cudaSuccess) return HGEMM_ERR_CUDA;
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return HGEMM_SUCCESS;
}

// k-blocks per stage of the streaming kernel (G): G > 1 fetches Bk through the
// 3-D k-block-grouped map (needs K % 64 == 0 and G | K/64) as long as at least
// 3 stages of G k-blocks still fit in shared memory (n = 128: G = 2 with 3 stages
// 32.8 us, G = 1 with 7 stages 34.8 us; profiles/r02/skinny_kgroup_ab.log).
int stream_kgroup(int64_t k, uint32_t a_bytes, int cw) {
  if (k % 64 != 0) return 1;
  const int64_t nkb = k / 64;
  int g = g_env_stream_g >= 1 ? g_env_stream_g : 2;
  const uint32_t kb_bytes = a_bytes + static_cast<uint32_t>(cw) * 128u;
  const uint32_t min_stages = g_env_stream_g >= 1 ? 2u : 3u;
  while (g > 1 && (nkb % g != 0 || (hg::kStreamSmemBytes - 1536u - 8192u) / (g * kb_bytes) < min_stages)) g /= 2;
  return g < 1 ? 1 : g;
}

// Chunk width for the streaming kernel: the smallest number of chunk waves over
// the SMs, then the widest chunk (fewest Ak re-reads) among those.
int stream_chunk(int64_t N, int mt, int num_sms) {
  const int cw_max = mt == 1 ? 256 : 128;
  int best = cw_max;
  int64_t best_w = INT64_MAX;
  for (int cw = cw_max; cw >= 16; cw -= 16) {
    const int64_t chunks = (N + cw - 1) / cw;
    const int64_t waves = (chunks + num_sms - 1) / num_sms;
    if (waves * cw < best_w) { best_w = waves * cw; best = cw; }
  }
  return best;
}

// The streaming kernel takes HBM-bound skinny shapes: M (= n) <= 256 with an
// N (= m) that gives every SM at least 4 chunk rows of 16.
// M <= 128 only: at M = 256 the two 16 KB Ak subtiles per k-block leave room for
// 4 stages (56 KB of HBM loads in flight per SM) and the CTA-pair tile kernel
// (256-wide tiles, 128 SMs) measured faster: 37.7 vs 44.2 us at 16384 x 256 x 4096
// (profiles/r02/skinny_kgroup_ab.log).
inline bool choose_stream(int64_t M, int64_t N, int64_t K, int num_sms) {
  return M <= g_env_stream_mmax && N >= static_cast<int64_t>(num_sms) * 64 && K >= 256;
}

// Swapped streaming (small m = Ms <= 256, long n = Ns) is available when forced
// (hgemm_config_t kernel = HGEMM_KERNEL_STREAM) but not chosen automatically: on
// the LSTM-gate shapes it measured slower than split-K (m = 64: 22.5 vs 14.4 us;
// m = 256: 30.7 vs 16.4 us; profiles/r01b/lstm_swapped_stream.log) -- each
// 32-row chunk re-reads the resident op(A) k-block by k-block and issues N = 32 MMAs.
inline bool choose_stream_swapped(int64_t, int64_t, int64_t, int) { return false; }

// One launch of the streaming kernel (hgemm_stream.cuh) on the resident operand
// R (Ms rows of k, K-contiguous, row pitch ldr; the UMMA A operand, Ak) and the
// streamed operand S (Ns rows, pitch lds; Bk): D (Ms x Ns) = R S^T, stored at C
// row-major with pitch ldc, or transposed (tout, the swapped-operand use).
hgemm_status_t run_stream(const void *R, int64_t ldr, int64_t Ms, const void *S, int64_t lds, int64_t Ns, int64_t k,
                          float alpha, float beta, void *C, int64_t ldc, bool f32, int tout, const hgemm_config_t &cfg,
                          int num_sms, int dev, cudaStream_t stream) {
  const int mt = Ms <= 128 ? 1 : 2;
  const bool forced_cw = cfg.kernel == HGEMM_KERNEL_STREAM && cfg.block_n;
  int cw = forced_cw ? cfg.block_n : stream_chunk(Ns, mt, num_sms);
  if (mt == 2 && cw > 128) cw = 128;
  // Ak TMA box rows (hgemm_stream.cuh): 64 when Ms <= 64 (the M = 128 MMA reads
  // 8 KB past the 64 real Ak rows: the next k-block, the stage's Bk or the pad)
  const uint32_t a_rows = (Ms <= 64) ? 64u : 128u;
  CUtensorMap ta, tb;
  const uint32_t a_bytes = a_rows == 64 ? 8192u : static_cast<uint32_t>(mt) * 16384u;
  const int kg = stream_kgroup(k, a_bytes, cw);
  // Ak through the 3-D k-group view as well (one row request per 256 B; MT == 1, G == 2)
  const int a3d = (mt == 1 && kg == 2 && g_env_stream_a3d) ? 1 : 0;
  bool ok = a3d ? make_map_3d(&ta, R, static_cast<uint64_t>(k), static_cast<uint64_t>(Ms), ldr, a_rows, 2)
                : make_map(&ta, R, static_cast<uint64_t>(k), static_cast<uint64_t>(Ms), ldr, 64, a_rows);
  if (ok) ok = kg > 1 ? make_map_3d(&tb, S, static_cast<uint64_t>(k), static_cast<uint64_t>(Ns), lds, cw, kg)
                      : make_map(&tb, S, static_cast<uint64_t>(k), static_cast<uint64_t>(Ns), lds, 64, cw);
  if (!ok) return HGEMM_ERR_CUDA;
  hg::StreamParams p = {};
  p.M = static_cast<int32_t>(Ms);
  p.N = static_cast<int32_t>(Ns);
  p.K = static_cast<int32_t>(k);
  p.cw = cw;
  p.num_chunks = static_cast<int32_t>(cdiv(Ns, cw));
  p.num_k_blocks = static_cast<int32_t>(cdiv(k, 64));
  p.a_bytes = a_bytes;
  p.kg = kg;
  p.b3d = kg > 1 ? 1 : 0;
  p.a3d = a3d;
  p.stage_bytes = static_cast<uint32_t>(kg) * (a_bytes + static_cast<uint32_t>(cw) * 128u);
  p.stages = static_cast<int32_t>(std::min<uint32_t>(
      hg::kStreamMaxStages, (hg::kStreamSmemBytes - 1536u - (a_rows == 64 ? 8192u : 0u)) / p.stage_bytes));
  if (g_env_stream_stages >= 2) p.stages = std::min(p.stages, g_env_stream_stages);
  p.probe = g_probe.load(std::memory_order_relaxed);
  p.k_rot = tout ? 1 : g_env_stream_rot;
  p.alpha = alpha;
  p.beta = beta;
  p.D = C;
  p.ldd = ldc;
  p.tout = tout;
  p.pre = std::max(1, std::min(p.stages, g_env_stream_pre > 0 ? g_env_stream_pre : p.stages));
  int grid = static_cast<int>(std::min<int64_t>(p.num_chunks, num_sms));
  if (cfg.max_ctas > 0) grid = std::min(grid, cfg.max_ctas);
  hgemm_status_t st;
  if (mt == 1) st = f32 ? launch_stream<1, true>(ta, tb, p, grid, dev, stream)
                        : launch_stream<1, false>(ta, tb, p, grid, dev, stream);
  else st = f32 ? launch_stream<2, true>(ta, tb, p, grid, dev, stream)
                : launch_stream<2, false>(ta, tb, p, grid, dev, stream);
  if (st == HGEMM_SUCCESS) {
    std::lock_guard<std::mutex> lk(g_mu);
    g_last = {HGEMM_KERNEL_STREAM, cw, tout /* 1: swapped */, grid, kg /* k-blocks per stage */, 0};
  }
  return st;
}

inline bool is_t(char c) { return c == 'T' || c == 't'; }
inline bool is_n(char c) { return c == 'N' || c == 'n'; }
inline bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// Relative per-SM throughput of a CTA-pair tile tn columns wide (flexible width, 256-wide
// kernel): the L2 -> SMEM demand per tensor cycle grows as the tile narrows (each CTA loads
// 16 KB of Ak + tn/2 rows of Bk per k-block for 512*tn/256 tensor cycles:
// 8192/tn + 32 B/clk/SM), so the efficiency falls below the 256-wide tile's 0.93.
inline double flex_eff(int tn) {
  const double demand = 8192.0 / tn + 32.0, demand256 = 8192.0 / 256 + 32.0;
  return 0.93 * std::pow(demand256 / demand, 0.5);
}

// Automatic tile choice: estimated time = waves * per-wave tile cost.  flex_ok: the
// 256-wide CTA-pair kernel may use a flexible tile width (K-major Bk); tn returns the
// chosen width (0: the kernel's own BN).
void choose_tc(int64_t M, int64_t N, int64_t K, bool beta_nonzero, int num_sms, int forced_cg, int sk_mode, int &cg,
               int &bn, bool flex_ok, int &tn, bool kg_ok) {
  struct Cand { int cg, bn, tn; double eff; };
  // eff: relative per-SM throughput of the tile shape.  Larger tiles move
  // fewer L2->SMEM bytes per FLOP (pair 256x512: 171 FLOP/B, 256x256: 128,
  // 1-SM 128x256: 85, 128x128: 64), which under the 1 kW power cap buys clock.
  Cand cands[16] = {{2, 512, 0, 1.00}, {2, 256, 0, 0.93}, {1, 256, 0, 0.85}, {1, 128, 0, 0.75}};
  int nc = 4;
  if (flex_ok)  // flexible widths 240, 224, ..., 144 for the CTA-pair 256-wide kernel
    for (int w = 240; w >= 144; w -= 16) cands[nc++] = {2, 256, w, flex_eff(w)};
  double best = 1e300;
  tn = 0;
  for (int ci = 0; ci < nc; ++ci) {
    const Cand &c = cands[ci];
    if (forced_cg && c.cg != forced_cg) continue;
    const int width = c.tn ? c.tn : c.bn;
    // One 512-column accumulator cannot fully overlap the epilogue with the
    // next tile's mainloop, and its staging (one box per epilogue warp) cannot
    // prefetch a whole accumulator half of C; with beta != 0 that costs ~3% at
    // K = 8192 and ~7% at K = 1024 (BERT-FFN shapes).
    double eff = (c.bn == 512 && beta_nonzero) ? (K < 4096 ? 0.90 : 0.97) : c.eff;
    // flexible tiles with beta != 0 take the chunked epilogue (C through registers)
    if (c.tn && beta_nonzero) eff *= 0.95;
    // 1-SM tiles with one k-block per stage need 0.75-1 TMA box rows per tensor cycle (128 B
    // each), far above what the TMA engine delivers (~0.3 rows/clk, profiles/r02/
    // l2_ingest_study.log); short k loops hide it in the fixed costs, long ones do not:
    // 1280 x 1280 x 5120 34.1 us with 128 x 128 tiles, 28.6 with CTA-pair 256-wide tiles +
    // stream-K.  The 128 x 128 tile with k-group stages (kg_ok: layout TN, k % 128 == 0) halves
    // its rows per cycle and beats both there (26.8 us; profiles/r02/chooser_probe.log).
    if (c.cg == 1 && cdiv(K, 64) >= 64 && !(kg_ok && c.bn == 128)) eff *= 0.65;
    const int64_t tiles = cdiv(M, 128 * c.cg) * cdiv(N, width);
    const int64_t units = num_sms / c.cg;
    double waves = static_cast<double>(cdiv(tiles, units));
    const int64_t nkb = cdiv(K, 64);
    // 512-wide: a last wave of r <= units/2 tiles after >= 4 whole waves runs as
    // 256-wide halves (launch_tc), measured ~0.6 of a wave
    const int ht_mode = sk_mode >> 4;
    if (c.bn == 512 && ht_mode != 1 && (sk_mode & 15) != 2 && tiles % units != 0 &&
        2 * (tiles % units) <= units && (ht_mode == 2 || tiles / units >= 4))
      waves = static_cast<double>(tiles / units) + 0.6;
    // stream-K: fractional waves (256-wide tiles only: with 512-wide tiles the FP32
    // partials of a split tile are twice as large and it measured slower everywhere)
    if (c.bn <= 256 && !c.tn && sk_plan(tiles, units, nkb, sk_mode & 15) >= 0)
      waves = static_cast<double>(tiles) / units + sk_overhead_waves(nkb);
    const double t = waves * (128.0 * c.cg * width) / (c.cg * eff);
    if (t < best * 0.999) { best = t; cg = c.cg; bn = c.bn; tn = c.tn; }
  }
}

}  // namespace

extern "C" {

const char *hgemm_status_string(hgemm_status_t s) {
  switch (s) {
    case HGEMM_SUCCESS: return "HGEMM_SUCCESS";
    case HGEMM_ERR_INVALID_VALUE: return "HGEMM_ERR_INVALID_VALUE: invalid argument";
    case HGEMM_ERR_ARCH: return "HGEMM_ERR_ARCH: device is not compute capability 10.0 (sm_100a)";
    case HGEMM_ERR_CUDA: return "HGEMM_ERR_CUDA: CUDA runtime/driver error";
  }
  return "HGEMM: unknown status";
}

hgemm_status_t hgemm_set_config(const hgemm_config_t *cfg) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!cfg) {
    g_cfg = {HGEMM_KERNEL_AUTO, 0, 0, 0, 0, 0, 0, 0};
    return HGEMM_SUCCESS;
  }
  if (cfg->kernel < HGEMM_KERNEL_AUTO || cfg->kernel > HGEMM_KERNEL_STREAM) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->stream_k < 0 || cfg->stream_k > 2) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->half_tail < 0 || cfg->half_tail > 2) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->kernel == HGEMM_KERNEL_SPLITK) {
    if (cfg->block_n != 0 && cfg->block_n != 64 && cfg->block_n != 128) return HGEMM_ERR_INVALID_VALUE;
    if (cfg->splits != 0 && cfg->splits != 2 && cfg->splits != 4 && cfg->splits != 8) return HGEMM_ERR_INVALID_VALUE;
    if (cfg->group_m < 0 || cfg->max_ctas < 0) return HGEMM_ERR_INVALID_VALUE;
    g_cfg = *cfg;
    return HGEMM_SUCCESS;
  }
  if (cfg->splits != 0) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->tile_n != 0 && cfg->kernel != HGEMM_KERNEL_TC_2SM) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->kernel == HGEMM_KERNEL_STREAM) {
    if (cfg->block_n < 0 || cfg->block_n > 256 || cfg->block_n % 16 != 0) return HGEMM_ERR_INVALID_VALUE;
    if (cfg->group_m < 0 || cfg->max_ctas < 0) return HGEMM_ERR_INVALID_VALUE;
    g_cfg = *cfg;
    return HGEMM_SUCCESS;
  }
  if (cfg->block_n != 0 && cfg->block_n != 128 && cfg->block_n != 256 && cfg->block_n != 512)
    return HGEMM_ERR_INVALID_VALUE;
  // flexible width: the CTA-pair 256-wide kernel only, a multiple of 16 in [128, 256]
  if (cfg->tile_n != 0 && (cfg->kernel != HGEMM_KERNEL_TC_2SM || cfg->block_n != 256 || cfg->tile_n % 16 != 0 ||
                           cfg->tile_n < 128 || cfg->tile_n > 256))
    return HGEMM_ERR_INVALID_VALUE;
  if (cfg->kernel == HGEMM_KERNEL_TC_2SM && cfg->block_n == 128) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->kernel == HGEMM_KERNEL_TC_1SM && cfg->block_n == 512) return HGEMM_ERR_INVALID_VALUE;
  if (cfg->group_m < 0 || cfg->max_ctas < 0) return HGEMM_ERR_INVALID_VALUE;
  g_cfg = *cfg;
  return HGEMM_SUCCESS;
}

hgemm_status_t hgemm_get_last_config(hgemm_config_t *out) {
  if (!out) return HGEMM_ERR_INVALID_VALUE;
  std::lock_guard<std::mutex> lk(g_mu);
  *out = g_last;
  return HGEMM_SUCCESS;
}

int64_t hgemm_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

hgemm_status_t hgemm_set_probe(unsigned long long *device_buf) {
  g_probe.store(device_buf, std::memory_order_relaxed);
  return HGEMM_SUCCESS;
}

}  // extern "C"

namespace {

// Fused all-gather of op(A) (hgemm_allgather_a): the kernel waits per chunk of
// op(A) rows for the copy stream's flag; raster groups along N, one group per
// chunk, starting with the group of this rank's first local chunk.
struct AgSpec {
  int *ctr;                 // [0] work index, [1 + c] finished copy units of chunk c (zeroed)
  const void *const *peers;
  const int64_t *rs;
  int world, rank;
  int64_t chunk_rows, unit_rows, units;
};

hgemm_status_t hgemm_core(int64_t m, int64_t n, int64_t k, float alpha, const void *A, int64_t lda,
                          const void *B, int64_t ldb, float beta, void *C, int64_t ldc, char transA, char transB,
                          hgemm_dtype_t out_dtype, cudaStream_t stream, const AgSpec *ag, bool acc16 = false) {
  // ---------------------------------------------------------- validation (no side effects)
  if (m < 0 || n < 0 || k < 0) return HGEMM_ERR_INVALID_VALUE;
  if (!(is_t(transA) || is_n(transA)) || !(is_t(transB) || is_n(transB))) return HGEMM_ERR_INVALID_VALUE;
  if (out_dtype != HGEMM_OUT_F16 && out_dtype != HGEMM_OUT_F32) return HGEMM_ERR_INVALID_VALUE;
  if (acc16 && (out_dtype != HGEMM_OUT_F16 || ag)) return HGEMM_ERR_INVALID_VALUE;
  const bool tA = is_t(transA), tB = is_t(transB);
  if (lda < std::max<int64_t>(1, tA ? k : m)) return HGEMM_ERR_INVALID_VALUE;
  if (ldb < std::max<int64_t>(1, tB ? n : k)) return HGEMM_ERR_INVALID_VALUE;
  if (ldc < std::max<int64_t>(1, m)) return HGEMM_ERR_INVALID_VALUE;
  if (m == 0 || n == 0) {
    std::lock_guard<std::mutex> lk(g_mu);
    g_last = {HGEMM_KERNEL_AUTO, 0, 0, 0, 0};
    return HGEMM_SUCCESS;
  }
  if (!C) return HGEMM_ERR_INVALID_VALUE;
  const bool need_ab = (k > 0 && alpha != 0.0f);
  if (need_ab && (!A || !B)) return HGEMM_ERR_INVALID_VALUE;

  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return HGEMM_ERR_CUDA;
  DeviceInfo di;
  if (!device_info(dev, di)) return HGEMM_ERR_CUDA;
  if (!di.ok) return HGEMM_ERR_ARCH;
  const bool f32 = (out_dtype == HGEMM_OUT_F32);
  hgemm_config_t cfg;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    cfg = g_cfg;
  }

  // ---------------------------------------------------------- BLAS quick return: C = beta*C
  if (!need_ab) {
    const int64_t total = m * n;
    const int threads = 256;
    const int64_t blocks = std::min<int64_t>(cdiv(total, threads), static_cast<int64_t>(di.num_sms) * 8);
    if (f32) hg::hgemm_scale_kernel<true><<<static_cast<unsigned>(blocks), threads, 0, stream>>>(m, n, beta, C, ldc);
    else hg::hgemm_scale_kernel<false><<<static_cast<unsigned>(blocks), threads, 0, stream>>>(m, n, beta, C, ldc);
    if (cudaPeekAtLastError() != cudaSuccess) return HGEMM_ERR_CUDA;
    g_launches.fetch_add(1, std::memory_order_relaxed);
    std::lock_guard<std::mutex> lk(g_mu);
    g_last = {HGEMM_KERNEL_AUTO, 0, 0, 0, 0};
    return HGEMM_SUCCESS;
  }

  // ---------------------------------------------------------- fast-path preconditions
  const int out_size = f32 ? 4 : 2;
  const bool tc_ok = aligned16(A) && aligned16(B) && aligned16(C) && (lda % 8 == 0) && (ldb % 8 == 0) &&
                     ((ldc * out_size) % 16 == 0) && m < (1ll << 31) && n < (1ll << 31) && k < (1ll << 31) &&
                     lda < (1ll << 36) && ldb < (1ll << 36) && ldc < (1ll << 36) && encode_fn() != nullptr;
  const bool want_simt = !ag && (cfg.kernel == HGEMM_KERNEL_SIMT);
  if (!tc_ok || want_simt) {
    // grid.y is limited to 65535 blocks of 64 columns: wider problems run as several
    // launches over column ranges (pointer offsets into op(B) and C)
    constexpr int64_t kColsPerLaunch = 65535ll * 64;
    for (int64_t j0 = 0; j0 < n; j0 += kColsPerLaunch) {
      const int64_t nj = std::min(n - j0, kColsPerLaunch);
      dim3 grid(static_cast<unsigned>(cdiv(m, 64)), static_cast<unsigned>(cdiv(nj, 64)));
      const __half *Ah = static_cast<const __half *>(A);
      const __half *Bh = static_cast<const __half *>(B);
      if (Bh) Bh += tB ? j0 : j0 * ldb;
      void *Cj = static_cast<char *>(C) + j0 * ldc * (f32 ? 4 : 2);
      if (f32) hg::hgemm_simt_kernel<true, false><<<grid, 256, 0, stream>>>(m, nj, k, alpha, Ah, lda, Bh, ldb, beta, Cj, ldc, tA, tB);
      else if (acc16) hg::hgemm_simt_kernel<false, true><<<grid, 256, 0, stream>>>(m, nj, k, alpha, Ah, lda, Bh, ldb, beta, Cj, ldc, tA, tB);
      else hg::hgemm_simt_kernel<false, false><<<grid, 256, 0, stream>>>(m, nj, k, alpha, Ah, lda, Bh, ldb, beta, Cj, ldc, tA, tB);
      if (cudaPeekAtLastError() != cudaSuccess) return HGEMM_ERR_CUDA;
      g_launches.fetch_add(1, std::memory_order_relaxed);
    }
    std::lock_guard<std::mutex> lk(g_mu);
    g_last = {HGEMM_KERNEL_SIMT, 0, 0, 0, 0};
    return HGEMM_SUCCESS;
  }

  // ---------------------------------------------------------- tcgen05 path
  const int64_t M = n, N = m;  // kernel coordinates (D = C^T)
  const bool a_mn = tB;   // Ak = op(B)^T: 'T' -> rows of Ak contiguous along M
  const bool b_mn = !tA;  // Bk = op(A):   'N' -> rows of Bk contiguous along N

  // ---------------------------------------------------------- HBM streaming (skinny, TN)
  if (!ag && !acc16 && !a_mn && !b_mn && M <= 256 &&
      ((cfg.kernel == HGEMM_KERNEL_STREAM) ||
       (cfg.kernel == HGEMM_KERNEL_AUTO && choose_stream(M, N, k, di.num_sms))))
    return run_stream(B, ldb, M, A, lda, N, k, alpha, beta, C, ldc, f32, 0, cfg, di.num_sms, dev, stream);

  // ---------------------------------------------------------- HBM streaming, swapped operands
  // Small m with a long n (LSTM gates, batch <= 256): the big operand is op(B).  The
  // streaming kernel then keeps op(A) (m <= 256 rows) resident as its UMMA A operand,
  // streams the rows of op(B)^T (K-contiguous for transB 'N') and stores D = C
  // transposed (column-major C, element (i, j) at C + j*ldc + i).
  if (!ag && !acc16 && !a_mn && !b_mn && N <= 256 && M > 256 &&
      ((cfg.kernel == HGEMM_KERNEL_STREAM) ||
       (cfg.kernel == HGEMM_KERNEL_AUTO && choose_stream_swapped(N, M, k, di.num_sms))))
    return run_stream(A, lda, N, B, ldb, M, k, alpha, beta, C, ldc, f32, 1, cfg, di.num_sms, dev, stream);

  // ---------------------------------------------------------- split-K (under-filled shapes)
  {
    int sk_bn = 0, sk_spl = 0;
    bool use_sk = false, auto_hm = false;
    if (ag || acc16) {
      // the fused all-gather and FP16 accumulation run the persistent tile kernel only
    } else if (cfg.kernel == HGEMM_KERNEL_SPLITK) {
      use_sk = true;
      sk_bn = cfg.block_n ? cfg.block_n : (N <= 64 ? 64 : 128);
      sk_spl = cfg.splits ? cfg.splits : 4;
    } else if (cfg.kernel == HGEMM_KERNEL_AUTO) {
      use_sk = choose_splitk(M, N, k, di.num_sms, sk_bn, sk_spl, auto_hm);
    }
    // 64 x 64 tiles with 64 valid Ak rows (hgemm_splitk.cuh "HM"): twice the tiles, half the splits
    // (HGEMM_SK_HM=1, experiments: every 64-wide split-K launch, automatic ones with half the splits)
    const bool hm_ok = use_sk && sk_bn == 64 && g_env_sk_hm > 0;
    if (hm_ok && cfg.kernel == HGEMM_KERNEL_AUTO && sk_spl > 2 && !auto_hm) sk_spl /= 2;
    const bool sk_hm = (auto_hm || hm_ok) && (sk_spl == 2 || sk_spl == 4);
    if (use_sk) {
      CUtensorMap ta, tb;
      bool ok;
      const uint32_t a_box_rows = sk_hm ? 64u : 128u;
      // k-groups of 2 (3-D Ak view, one load of 256 contiguous bytes per Ak row): K-major Ak,
      // K % 64 == 0 and every split's k range a whole number of groups
      const int nkb_all = static_cast<int>(cdiv(k, 64));
      const int sk_kg = (!a_mn && k % 64 == 0 && nkb_all % (2 * sk_spl) == 0 && g_env_sk_kg == 2) ? 2 : 1;
      // op(A) (Bk) through the 3-D k-group view too: one row request per 256 B (DESIGN.md
      // "k-group loads in the tile kernel")
      const int sk_b3d = (sk_kg == 2 && !b_mn && g_env_sk_b3d) ? 1 : 0;
      if (!a_mn) ok = sk_kg == 2 ? make_map_3d(&ta, B, static_cast<uint64_t>(k), static_cast<uint64_t>(n), ldb, a_box_rows, 2)
                                 : make_map(&ta, B, static_cast<uint64_t>(k), static_cast<uint64_t>(n), ldb, 64, a_box_rows);
      else ok = make_map(&ta, B, static_cast<uint64_t>(n), static_cast<uint64_t>(k), ldb, 64, 64);
      if (ok) {
        if (!b_mn) ok = sk_b3d ? make_map_3d(&tb, A, static_cast<uint64_t>(k), static_cast<uint64_t>(m), lda, sk_bn, 2)
                               : make_map(&tb, A, static_cast<uint64_t>(k), static_cast<uint64_t>(m), lda, 64, sk_bn);
        else ok = make_map(&tb, A, static_cast<uint64_t>(m), static_cast<uint64_t>(k), lda, 64, 64);
      }
      if (!ok) return HGEMM_ERR_CUDA;
      TcParams p = {};
      p.M = static_cast<int32_t>(M);
      p.N = static_cast<int32_t>(N);
      p.K = static_cast<int32_t>(k);
      p.num_m_tiles = static_cast<int32_t>(cdiv(M, sk_hm ? 64 : 128));
      p.num_n_tiles = static_cast<int32_t>(cdiv(N, sk_bn));
      p.num_k_blocks = static_cast<int32_t>(cdiv(k, 64));
      p.group_m = p.num_m_tiles;  // tiles in m-fastest order
      p.sk_kg = sk_kg;
      p.sk_b3d = sk_b3d;
      p.alpha = alpha;
      p.beta = beta;
      p.D = C;
      p.ldd = ldc;
      p.probe = g_probe.load(std::memory_order_relaxed);
      const hgemm_status_t st = sk_bn == 64 ? hgi::dispatch_splitk64(sk_spl, a_mn, b_mn, f32, ta, tb, p, dev, stream, sk_hm)
                                            : hgi::dispatch_splitk128(sk_spl, a_mn, b_mn, f32, ta, tb, p, dev, stream);
      if (st == HGEMM_SUCCESS) {
        std::lock_guard<std::mutex> lk(g_mu);
        g_last = {HGEMM_KERNEL_SPLITK, sk_bn, p.group_m, 0, sk_spl};
      }
      return st;
    }
  }

  int cg = 2, bn = 512, tnf = 0;  // tnf: flexible tile width (0 = bn)
  // the fused all-gather and FP16-accumulate kernels exist for CTA pairs only
  const int forced_cg = (ag || acc16) ? 2 : cfg.kernel == HGEMM_KERNEL_TC_1SM ? 1 : cfg.kernel == HGEMM_KERNEL_TC_2SM ? 2 : 0;
  // stream-K is off under the fused all-gather (its work items do not follow the chunk order)
  // and with FP16 accumulation (no FP32 partials); stream-K mode with hgemm_config_t::half_tail
  // packed above it (launch_tc, choose_tc)
  const int skm = ((ag || acc16) ? 1 : cfg.stream_k) | (cfg.half_tail << 4);
  // flexible tile widths need a K-major Bk (TMA boxes of any multiple of 8 rows)
  const bool flex_ok = !b_mn && !ag && (skm & 15) != 2;
  if (forced_cg && cfg.block_n && !((ag || acc16) && cfg.block_n == 128)) {
    cg = forced_cg;
    bn = cfg.block_n;
    if (flex_ok && cg == 2 && bn == 256 && cfg.tile_n > 0 && cfg.tile_n < 256) tnf = cfg.tile_n;
  } else {
    // flexible widths are never chosen automatically: measured slower than the 256-wide tile
    // (with stream-K) at every mid-size shape tried (profiles/r02/flex_tile_sweep.log; DESIGN.md
    // "Flexible tile width"); the candidates stay available to the model for experiments
    choose_tc(M, N, k, beta != 0.0f, di.num_sms, forced_cg, skm, cg, bn, flex_ok && g_env_flex, tnf,
              g_env_tc_kg == 2 && g_env_tc1_kg && !a_mn && !b_mn && k % 128 == 0 && M > 256 && !ag && !acc16);
  }
  const int skm_eff = tnf ? ((skm & ~15) | 1) : skm;  // flexible tiles: whole tiles, no stream-K
  const int b_rows = (tnf ? tnf : (bn > 256 ? 256 : bn)) / cg;  // Bk rows per CTA per accumulator half
  // MC = 2: two CTA pairs per cluster share (multicast) the Bk half-boxes
  // (measured slower everywhere: a 4-CTA cluster strands SMs of the GPCs and couples
  // the two pairs' pipelines; built only with -DHGEMM_ENABLE_MC)
  int mc = 1;
#ifdef HGEMM_ENABLE_MC
  if (cg == 2 && !ag && !acc16) {
    mc = g_env_mc == 2 ? 2 : 1;  // experiments
  }
#endif

  // k-group stages (KG = 2: two k-blocks per ring stage, each operand one 3-D TMA box of
  // 256 contiguous bytes per row): 256-wide tiles, both operands K-major, K % 128 == 0, whole
  // tiles
  // Not where the launch would use stream-K (W = 2304 / 2560 / 4608: the 1-k-block stages with
  // stream-K measured faster) and not for one row of pair tiles (M <= 256: the skinny
  // HBM-streaming case, where 3 stages of 64 KB keep fewer bytes in flight than 6 of 32 KB);
  // profiles/r02/tc_kgroup_ab.log.
  const int64_t kg_tiles = cdiv(M, 256) * cdiv(N, 256);
  const bool kg2 = g_env_tc_kg == 2 && ((cg == 2 && bn == 256) || (cg == 1 && bn == 128 && g_env_tc1_kg)) &&
                   !a_mn && !b_mn && k % 128 == 0 && !tnf &&
                   !ag && !acc16 && !(cg == 2 && g_env_direct != 0) && M > 256 &&
                   (g_env_tc_kg_sk || sk_plan(kg_tiles, di.num_sms / 2, cdiv(k, 64), skm & 15) < 0);
  CUtensorMap ta, tb;
  bool ok;
  if (kg2) {
    ok = make_map_3d(&ta, B, static_cast<uint64_t>(k), static_cast<uint64_t>(n), ldb, 128, 2) &&
         make_map_3d(&tb, A, static_cast<uint64_t>(k), static_cast<uint64_t>(m), lda, static_cast<uint32_t>(b_rows), 2);
    // (mc == 2: each stage's whole Bk half-box comes from one pair, so the box keeps b_rows rows)
  } else {
    if (!a_mn) ok = make_map(&ta, B, static_cast<uint64_t>(k), static_cast<uint64_t>(n), ldb, 64, 128);
    else ok = make_map(&ta, B, static_cast<uint64_t>(n), static_cast<uint64_t>(k), ldb, 64, 64);
    if (ok) {
      if (!b_mn) ok = make_map(&tb, A, static_cast<uint64_t>(k), static_cast<uint64_t>(m), lda, 64, b_rows / mc);
      else ok = make_map(&tb, A, static_cast<uint64_t>(m), static_cast<uint64_t>(k), lda, 64, 64);
    }
  }
  // D = C^T row-major (N = m contiguous), stored in 32-row x 128-B swizzled boxes
  CUtensorMap td;
  if (ok) ok = make_map(&td, C, static_cast<uint64_t>(m), static_cast<uint64_t>(n), ldc, f32 ? 32 : 64, 32, f32);
  if (!ok) return HGEMM_ERR_CUDA;

  TcParams p = {};
  p.M = static_cast<int32_t>(M);
  p.N = static_cast<int32_t>(N);
  p.K = static_cast<int32_t>(k);
  p.num_m_tiles = static_cast<int32_t>(cdiv(M, 128 * cg * mc));
  p.num_n_tiles = static_cast<int32_t>(cdiv(N, tnf ? tnf : bn));
  p.tile_n = tnf;
  p.num_k_blocks = static_cast<int32_t>(cdiv(k, 64));
  p.group_m = cfg.group_m > 0 ? cfg.group_m : 16 / mc;  // measured best with 256x512 pair tiles (profiles/)

  p.group_m = std::max(1, std::min(p.group_m, p.num_m_tiles));
  if (g_env_group_n > 0)  // experiments: group along N instead
    p.group_m = -std::max(1, std::min(g_env_group_n, p.num_n_tiles));
  p.l2_hint = g_env_l2_hint;
  p.exp_flags = g_env_exp;
  if (ag) {
    p.ag_ctr = ag->ctr;
    for (int q = 0; q < ag->world; ++q) p.ag_peer[q] = ag->peers[q];
    for (int q = 0; q <= ag->world; ++q) p.ag_rs[q] = ag->rs[q];
    p.ag_A = const_cast<void *>(A);
    p.ag_lda = lda;
    p.ag_world = ag->world;
    p.ag_rank = ag->rank;
    p.ag_chunk_rows = static_cast<int32_t>(ag->chunk_rows);
    p.ag_unit_rows = static_cast<int32_t>(ag->unit_rows);
    p.ag_units = static_cast<int32_t>(ag->units);
    // one raster group per chunk (bn-aligned chunks tiling N exactly), starting with
    // this rank's first chunk, so the tiles run in the order the copies complete
    if (ag->chunk_rows % bn == 0) {
      const int gn = static_cast<int>(ag->chunk_rows / bn);
      if (gn <= p.num_n_tiles && p.num_n_tiles % gn == 0) {
        p.group_m = -gn;
        p.n_rot = static_cast<int32_t>((ag->rs[ag->rank] / ag->chunk_rows) % (p.num_n_tiles / gn));
      }
    }
  }
  p.probe = g_probe.load(std::memory_order_relaxed);
  p.alpha = alpha;
  p.beta = beta;
  p.D = C;
  p.ldd = ldc;

  bool sk_used = false;
  const hgi::TcLaunch L = {&ta, &tb, &td, &p, dev, &di, cfg.max_ctas, skm_eff, &sk_used, stream};
  hgemm_status_t st;
  if (kg2) st = hgi::dispatch_tc256_kg2(cg, f32, L, mc);
  else if (cg == 2 && bn == 512) st = hgi::dispatch_tc512(mc, ag != nullptr, acc16, a_mn, b_mn, f32, L);
  else if (cg == 2)
    st = hgi::dispatch_tc256x2(mc, ag != nullptr, acc16, a_mn, b_mn, f32, L, g_env_direct != 0 && !tnf);
  else st = hgi::dispatch_tc1(bn, a_mn, b_mn, f32, L);
  if (st == HGEMM_SUCCESS) {
    std::lock_guard<std::mutex> lk(g_mu);
    g_last = {cg == 2 ? HGEMM_KERNEL_TC_2SM : HGEMM_KERNEL_TC_1SM, bn, p.group_m, cfg.max_ctas, kg2 ? 2 : 0,
              sk_used ? 2 : 1, t_half_used ? 2 : 1, tnf};  // splits: k-blocks per ring stage when 2 (KG)
  }
  return st;
}

}  // namespace

extern "C" {

hgemm_status_t hgemm(int64_t m, int64_t n, int64_t k, float alpha, const void *A, int64_t lda, const void *B,
                     int64_t ldb, float beta, void *C, int64_t ldc, char transA, char transB,
                     hgemm_dtype_t out_dtype, cudaStream_t stream) {
  return hgemm_core(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA, transB, out_dtype, stream, nullptr);
}

hgemm_status_t hgemm_ex(int64_t m, int64_t n, int64_t k, float alpha, const void *A, int64_t lda, const void *B,
                        int64_t ldb, float beta, void *C, int64_t ldc, char transA, char transB,
                        hgemm_dtype_t out_dtype, hgemm_compute_t compute, cudaStream_t stream) {
  if (compute != HGEMM_COMPUTE_F32 && compute != HGEMM_COMPUTE_F16) return HGEMM_ERR_INVALID_VALUE;
  return hgemm_core(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA, transB, out_dtype, stream, nullptr,
                    compute == HGEMM_COMPUTE_F16);
}

}  // extern "C"

// ===================================================================== host-buffer path
namespace {

struct HostPipe {
  bool init = false;
  cudaStream_t s_in = nullptr, s_comp = nullptr, s_out = nullptr;
  static constexpr int kEv = 64;
  cudaEvent_t ev_in[kEv] = {}, ev_comp[kEv] = {}, ev_start = nullptr;
};
HostPipe g_pipe[kMaxDevices];
std::mutex g_pipe_mu;                     // creation of the per-device pipeline
std::mutex g_pipe_call_mu[kMaxDevices];   // one hgemm_host call at a time per device

inline int64_t align_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

struct HostLayout {
  int64_t a_rows, a_cols, b_rows, b_cols;  // stored shapes
  int64_t off_a, off_b, off_c, total;      // workspace offsets (bytes)
};

HostLayout host_layout(int64_t m, int64_t n, int64_t k, bool tA, bool tB, bool f32) {
  HostLayout L;
  L.a_rows = tA ? k : m;
  L.a_cols = tA ? m : k;
  L.b_rows = tB ? n : k;
  L.b_cols = tB ? k : n;
  // device copies keep a 16-byte aligned pitch (the TMA fast-path precondition)
  const int64_t lda_d = align_up(std::max<int64_t>(L.a_rows, 1), 8);
  const int64_t ldb_d = align_up(std::max<int64_t>(L.b_rows, 1), 8);
  const int64_t ldc_d = align_up(std::max<int64_t>(m, 1), f32 ? 4 : 8);
  L.off_a = 0;
  L.off_b = align_up(L.off_a + lda_d * L.a_cols * 2, 256);
  L.off_c = align_up(L.off_b + ldb_d * L.b_cols * 2, 256);
  L.total = align_up(L.off_c + ldc_d * n * (f32 ? 4 : 2), 256);
  return L;
}

}  // namespace

extern "C" {

size_t hgemm_host_workspace_size(int64_t m, int64_t n, int64_t k, char transA, char transB,
                                 hgemm_dtype_t out_dtype) {
  if (m < 0 || n < 0 || k < 0) return 0;
  return static_cast<size_t>(host_layout(m, n, k, is_t(transA), is_t(transB), out_dtype == HGEMM_OUT_F32).total);
}

hgemm_status_t hgemm_host(int64_t m, int64_t n, int64_t k, float alpha, const void *A, int64_t lda, const void *B,
                          int64_t ldb, float beta, void *C, int64_t ldc, char transA, char transB,
                          hgemm_dtype_t out_dtype, void *workspace, size_t workspace_bytes, cudaStream_t stream) {
  if (m < 0 || n < 0 || k < 0) return HGEMM_ERR_INVALID_VALUE;
  if (!(is_t(transA) || is_n(transA)) || !(is_t(transB) || is_n(transB))) return HGEMM_ERR_INVALID_VALUE;
  if (out_dtype != HGEMM_OUT_F16 && out_dtype != HGEMM_OUT_F32) return HGEMM_ERR_INVALID_VALUE;
  const bool tA = is_t(transA), tB = is_t(transB), f32 = (out_dtype == HGEMM_OUT_F32);
  if (lda < std::max<int64_t>(1, tA ? k : m)) return HGEMM_ERR_INVALID_VALUE;
  if (ldb < std::max<int64_t>(1, tB ? n : k)) return HGEMM_ERR_INVALID_VALUE;
  if (ldc < std::max<int64_t>(1, m)) return HGEMM_ERR_INVALID_VALUE;
  if (m == 0 || n == 0) return HGEMM_SUCCESS;
  if (!C) return HGEMM_ERR_INVALID_VALUE;
  const bool need_ab = (k > 0 && alpha != 0.0f);
  if (need_ab && (!A || !B)) return HGEMM_ERR_INVALID_VALUE;
  const HostLayout L = host_layout(m, n, k, tA, tB, f32);
  if (!workspace || workspace_bytes < static_cast<size_t>(L.total)) return HGEMM_ERR_INVALID_VALUE;

  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return HGEMM_ERR_CUDA;
  HostPipe &P = g_pipe[dev];
  {
    std::lock_guard<std::mutex> lk(g_pipe_mu);
    if (!P.init) {
      if (cudaStreamCreateWithFlags(&P.s_in, cudaStreamNonBlocking) != cudaSuccess ||
          cudaStreamCreateWithFlags(&P.s_comp, cudaStreamNonBlocking) != cudaSuccess ||
          cudaStreamCreateWithFlags(&P.s_out, cudaStreamNonBlocking) != cudaSuccess ||
          cudaEventCreateWithFlags(&P.ev_start, cudaEventDisableTiming) != cudaSuccess)
        return HGEMM_ERR_CUDA;
      for (int i = 0; i < HostPipe::kEv; ++i)
        if (cudaEventCreateWithFlags(&P.ev_in[i], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&P.ev_comp[i], cudaEventDisableTiming) != cudaSuccess)
          return HGEMM_ERR_CUDA;
      P.init = true;
    }
  }
  // the pipeline streams/events of a device serve one call at a time (calls on other devices proceed)
  std::lock_guard<std::mutex> call_lk(g_pipe_call_mu[dev]);
  const int esz = f32 ? 4 : 2;
  uint8_t *ws = static_cast<uint8_t *>(workspace);
  const int64_t lda_d = align_up(std::max<int64_t>(L.a_rows, 1), 8);
  const int64_t ldb_d = align_up(std::max<int64_t>(L.b_rows, 1), 8);
  const int64_t ldc_d = align_up(std::max<int64_t>(m, 1), f32 ? 4 : 8);
  uint8_t *dA = ws + L.off_a, *dB = ws + L.off_b, *dC = ws + L.off_c;
  const uint8_t *hA = static_cast<const uint8_t *>(A), *hB = static_cast<const uint8_t *>(B);
  uint8_t *hC = static_cast<uint8_t *>(C);

  // Column panels of op(B)/C (>= 1024 columns, at most 8, a multiple of 256 wide).  The
  // first panel's GEMM is further cut into row pieces of op(A) (multiples of 256 rows) so
  // that it starts once the first piece of A has arrived instead of all of A.
  int64_t panels = std::min<int64_t>(8, std::max<int64_t>(1, n / 1024));
  const int64_t pw = align_up(cdiv(n, panels), 256);
  panels = cdiv(n, pw);
  const int64_t pieces = need_ab ? std::min<int64_t>(4, std::max<int64_t>(1, m / 2048)) : 1;
  const int64_t ph = align_up(cdiv(m, pieces), 256);

  // Once anything is enqueued, an error return first drains the internal streams: no
  // copy may still read or write the caller's host buffers after the call returns.
  auto fail = [&](hgemm_status_t st) {
    cudaStreamSynchronize(P.s_in);
    cudaStreamSynchronize(P.s_comp);
    cudaStreamSynchronize(P.s_out);
    return st;
  };
  int step = 0;
  // one pipeline step: (H2D copies already on s_in) -> GEMM of C[r0:r1, n0:n1] on s_comp -> D2H on s_out
  auto gemm_step = [&](int64_t r0, int64_t r1, int64_t n0, int64_t n1) -> hgemm_status_t {
    if (cudaEventRecord(P.ev_in[step], P.s_in) != cudaSuccess) return HGEMM_ERR_CUDA;
    if (cudaStreamWaitEvent(P.s_comp, P.ev_in[step], 0) != cudaSuccess) return HGEMM_ERR_CUDA;
    const uint8_t *dAi = dA + (tA ? r0 * lda_d : r0) * 2;
    const uint8_t *dBj = dB + (tB ? n0 : n0 * ldb_d) * 2;
    uint8_t *dCij = dC + (r0 + n0 * ldc_d) * esz;
    const hgemm_status_t st = hgemm(r1 - r0, n1 - n0, k, alpha, dAi, lda_d, dBj, ldb_d, beta, dCij, ldc_d, transA,
                                    transB, out_dtype, P.s_comp);
    if (st != HGEMM_SUCCESS) return st;
    if (cudaEventRecord(P.ev_comp[step], P.s_comp) != cudaSuccess) return HGEMM_ERR_CUDA;
    if (cudaStreamWaitEvent(P.s_out, P.ev_comp[step], 0) != cudaSuccess) return HGEMM_ERR_CUDA;
    if (cudaMemcpy2DAsync(hC + (r0 + n0 * ldc) * esz, ldc * esz, dCij, ldc_d * esz, (r1 - r0) * esz, n1 - n0,
                          cudaMemcpyDeviceToHost, P.s_out) != cudaSuccess)
      return HGEMM_ERR_CUDA;
    ++step;
    return HGEMM_SUCCESS;
  };
  auto copy_b = [&](int64_t n0, int64_t n1) -> bool {  // op(B)[:, n0:n1] (+ C[:, n0:n1] when beta != 0)
    const int64_t w = n1 - n0;
    if (need_ab) {
      // B columns (transB 'N') or B rows (transB 'T')
      const size_t width = static_cast<size_t>(tB ? w : L.b_rows) * 2;
      const size_t height = static_cast<size_t>(tB ? L.b_cols : w);
      if (cudaMemcpy2DAsync(dB + (tB ? n0 : n0 * ldb_d) * 2, ldb_d * 2, hB + (tB ? n0 : n0 * ldb) * 2, ldb * 2,
                            width, height, cudaMemcpyHostToDevice, P.s_in) != cudaSuccess)
        return false;
    }
    if (beta != 0.0f &&
        cudaMemcpy2DAsync(dC + n0 * ldc_d * esz, ldc_d * esz, hC + n0 * ldc * esz, ldc * esz, m * esz, w,
                          cudaMemcpyHostToDevice, P.s_in) != cudaSuccess)
      return false;
    return true;
  };

  if (cudaEventRecord(P.ev_start, stream) != cudaSuccess) return HGEMM_ERR_CUDA;
  if (cudaStreamWaitEvent(P.s_in, P.ev_start, 0) != cudaSuccess) return HGEMM_ERR_CUDA;
  if (!copy_b(0, std::min(n, pw))) return fail(HGEMM_ERR_CUDA);
  for (int64_t i = 0; i < pieces; ++i) {
    const int64_t r0 = i * ph, r1 = std::min(m, r0 + ph);
    if (r0 >= r1) break;
    if (need_ab) {
      // op(A)[r0:r1, :]: stored columns r0..r1 (transA 'T') or rows r0..r1 of every column ('N')
      const size_t width = static_cast<size_t>(tA ? L.a_rows : r1 - r0) * 2;
      const size_t height = static_cast<size_t>(tA ? r1 - r0 : L.a_cols);
      if (cudaMemcpy2DAsync(dA + (tA ? r0 * lda_d : r0) * 2, lda_d * 2, hA + (tA ? r0 * lda : r0) * 2, lda * 2,
                            width, height, cudaMemcpyHostToDevice, P.s_in) != cudaSuccess)
        return fail(HGEMM_ERR_CUDA);
    }
    const hgemm_status_t st = gemm_step(r0, r1, 0, std::min(n, pw));
    if (st != HGEMM_SUCCESS) return fail(st);
  }
  for (int64_t j = 1; j < panels; ++j) {
    const int64_t n0 = j * pw, n1 = std::min(n, n0 + pw);
    // the last panel goes in up to 4 slices (>= 256 columns each): only the last slice's GEMM
    // and device->host copy remain after the final host->device copy (the pipeline's tail)
    const int64_t slices = (j == panels - 1 && panels > 1) ? std::max<int64_t>(1, std::min<int64_t>(4, (n1 - n0) / 256)) : 1;
    const int64_t sw = align_up(cdiv(n1 - n0, slices), 8);
    for (int64_t s0 = n0; s0 < n1; s0 += sw) {
      const int64_t s1 = std::min(n1, s0 + sw);
      if (!copy_b(s0, s1)) return fail(HGEMM_ERR_CUDA);
      const hgemm_status_t st = gemm_step(0, m, s0, s1);
      if (st != HGEMM_SUCCESS) return fail(st);
    }
  }
  // make `stream` observe the end of the pipeline (events recorded on it bracket the whole call)
  if (cudaEventRecord(P.ev_comp[HostPipe::kEv - 1], P.s_out) != cudaSuccess) return fail(HGEMM_ERR_CUDA);
  if (cudaStreamWaitEvent(stream, P.ev_comp[HostPipe::kEv - 1], 0) != cudaSuccess) return fail(HGEMM_ERR_CUDA);
  if (cudaStreamSynchronize(P.s_out) != cudaSuccess) return fail(HGEMM_ERR_CUDA);
  return HGEMM_SUCCESS;
}

}  // extern "C"

// ============================================================================
// Sharded path: all-gather of op(A) fused with the GEMM (include/hgemm.h;
// BASELINE.json north_star (3), DESIGN.md "Fused
// all-gather").  An extra copy warp in every CTA of the persistent GEMM kernel
// pulls the peers' rows of op(A) over NVLink (16-B loads from P2P-mapped peer
// memory, 16 in flight per lane) into the local gather buffer, one ~64 KB copy
// unit at a time from a shared work index, and counts finished units per
// chunk; the TMA producer waits per tile for the chunks it reads.  The copy
// warp costs issue slots and registers next to the epilogue warps of its SM;
// the copy engines were rejected (a same-device cudaMemcpyAsync can run as a
// kernel that never becomes resident next to the persistent GEMM),
// and no NCCL kernel has to share the SMs with the GEMM.
namespace {

bool plan_args_ok(int64_t m, const int64_t *row_splits, int32_t world, int32_t rank, int64_t chunk_rows) {
  if (m < 0 || world < 1 || rank < 0 || rank >= world || chunk_rows < 1 || !row_splits) return false;
  if (row_splits[0] != 0 || row_splits[world] != m) return false;
  for (int q = 0; q < world; ++q)
    if (row_splits[q + 1] < row_splits[q]) return false;
  return true;
}

int owner_of(int64_t row, const int64_t *row_splits, int32_t world) {
  int q = 0;
  while (q + 1 < world && row >= row_splits[q + 1]) ++q;
  return q;
}

// Issue order: chunks grouped by the owner of their first row, owners in the
// order rank, rank+1, ... (mod world) so the local chunks come first and the
// ranks pull from different peers at any moment; within a chunk one record per
// owner segment.
template <typename F>
void plan_walk(int64_t m, const int64_t *row_splits, int32_t world, int32_t rank, int64_t chunk_rows, F &&emit) {
  const int64_t nchunks = (m + chunk_rows - 1) / chunk_rows;
  for (int d = 0; d < world; ++d) {
    const int q = (rank + d) % world;
    for (int64_t c = 0; c < nchunks; ++c) {
      const int64_t c0 = c * chunk_rows, c1 = std::min(m, c0 + chunk_rows);
      if (owner_of(c0, row_splits, world) != q) continue;
      int64_t r = c0;
      while (r < c1) {
        const int o = owner_of(r, row_splits, world);
        const int64_t e = std::min(c1, row_splits[o + 1]);
        emit(c, o, r, e);
        r = e;
      }
    }
  }
}

using MemGetAddressRangeFn = CUresult (*)(CUdeviceptr *, size_t *, CUdeviceptr);

template <typename Fn>
Fn driver_fn(const char *name) {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPointByVersion(name, &p, 12000, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return nullptr;
  return reinterpret_cast<Fn>(p);
}

struct IpcMapping {
  void *user;
  void *base;
};
std::mutex g_ipc_mu;
IpcMapping g_ipc[256];
int g_ipc_n = 0;

}  // namespace

extern "C" {

hgemm_status_t hgemm_allgather_plan(int64_t m, const int64_t *row_splits, int32_t world, int32_t rank,
                                    int64_t chunk_rows, int64_t *ops, int64_t max_ops, int64_t *num_ops) {
  if (!num_ops || !plan_args_ok(m, row_splits, world, rank, chunk_rows)) return HGEMM_ERR_INVALID_VALUE;
  int64_t cnt = 0;
  plan_walk(m, row_splits, world, rank, chunk_rows, [&](int64_t c, int o, int64_t r0, int64_t r1) {
    if (ops && cnt < max_ops) {
      ops[4 * cnt + 0] = c;
      ops[4 * cnt + 1] = o;
      ops[4 * cnt + 2] = r0;
      ops[4 * cnt + 3] = r1;
    }
    ++cnt;
  });
  *num_ops = cnt;
  return HGEMM_SUCCESS;
}

hgemm_status_t hgemm_allgather_a(int64_t m, int64_t n, int64_t k, float alpha, void *A, int64_t lda,
                                 const void *const *A_peers, const int64_t *row_splits, int32_t world, int32_t rank,
                                 const void *B, int64_t ldb, float beta, void *C, int64_t ldc, char transB,
                                 hgemm_dtype_t out_dtype, int32_t *workspace, int64_t workspace_ints,
                                 int64_t chunk_rows, cudaStream_t stream) {
  // ---------------------------------------------------------- validation (no side effects)
  if (m < 0 || n < 0 || k < 0) return HGEMM_ERR_INVALID_VALUE;
  if (!(is_t(transB) || is_n(transB))) return HGEMM_ERR_INVALID_VALUE;
  if (out_dtype != HGEMM_OUT_F16 && out_dtype != HGEMM_OUT_F32) return HGEMM_ERR_INVALID_VALUE;
  if (lda < std::max<int64_t>(1, k)) return HGEMM_ERR_INVALID_VALUE;
  if (ldb < std::max<int64_t>(1, is_t(transB) ? n : k)) return HGEMM_ERR_INVALID_VALUE;
  if (ldc < std::max<int64_t>(1, m)) return HGEMM_ERR_INVALID_VALUE;
  if (!plan_args_ok(m, row_splits, world, rank, chunk_rows)) return HGEMM_ERR_INVALID_VALUE;
  const int64_t nchunks = (m + chunk_rows - 1) / chunk_rows;
  if (!workspace || workspace_ints < 1 + nchunks) return HGEMM_ERR_INVALID_VALUE;
  if (m > 0 && k > 0 && !A) return HGEMM_ERR_INVALID_VALUE;
  for (int q = 0; q < world; ++q)
    if (q != rank && row_splits[q + 1] > row_splits[q] && k > 0 && (!A_peers || !A_peers[q]))
      return HGEMM_ERR_INVALID_VALUE;
  if (m > 0 && n > 0 && !C) return HGEMM_ERR_INVALID_VALUE;
  if (m > 0 && n > 0 && k > 0 && alpha != 0.0f && !B) return HGEMM_ERR_INVALID_VALUE;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return HGEMM_ERR_CUDA;
  DeviceInfo di;
  if (!device_info(dev, di)) return HGEMM_ERR_CUDA;
  if (!di.ok) return HGEMM_ERR_ARCH;

  // ---------------------------------------------------------- fused: one kernel gathers and multiplies
  const bool f32 = (out_dtype == HGEMM_OUT_F32);
  const int out_size = f32 ? 4 : 2;
  bool aligned_shards = world <= 8;
  for (int q = 1; q < world && aligned_shards; ++q)
    if (row_splits[q] % chunk_rows != 0 && row_splits[q] != m) aligned_shards = false;
  bool peers_aligned = true;
  for (int q = 0; q < world; ++q)
    if (q != rank && A_peers && !aligned16(A_peers[q])) peers_aligned = false;
  const bool fused = aligned_shards && peers_aligned && m > 0 && n > 0 && k > 0 && alpha != 0.0f && (k % 8 == 0) &&
                     aligned16(A) && aligned16(B) && aligned16(C) && (lda % 8 == 0) && (ldb % 8 == 0) &&
                     ((ldc * out_size) % 16 == 0) && m < (1ll << 31) && n < (1ll << 31) && k < (1ll << 31) &&
                     lda < (1ll << 36) && ldb < (1ll << 36) && ldc < (1ll << 36) && chunk_rows < (1ll << 30) &&
                     encode_fn() != nullptr;
  if (fused) {
    // copy unit: ~64 KB of rows, a power of two dividing chunk_rows (never straddles a chunk)
    const int64_t target = std::max<int64_t>(1, 65536 / (k * 2));
    int64_t u = 1;
    while (u * 2 <= target && chunk_rows % (u * 2) == 0) u *= 2;
    int64_t units = 0;
    for (int q = 0; q < world; ++q)
      if (q != rank) units += (row_splits[q + 1] - row_splits[q] + u - 1) / u;
    if (units < (1ll << 31)) {
      if (cudaMemsetAsync(workspace, 0, static_cast<size_t>(1 + nchunks) * 4, stream) != cudaSuccess)
        return HGEMM_ERR_CUDA;
      const AgSpec ag = {workspace, A_peers, row_splits, world, rank, chunk_rows, u, units};
      return hgemm_core(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, 'T', transB, out_dtype, stream, &ag);
    }
  }

  // ---------------------------------------------------------- unfused: copies, then hgemm()
  const size_t pitch = static_cast<size_t>(lda) * 2;
  hgemm_status_t st = HGEMM_SUCCESS;
  if (k > 0) {
    plan_walk(m, row_splits, world, rank, chunk_rows, [&](int64_t, int o, int64_t r0, int64_t r1) {
      if (st != HGEMM_SUCCESS || o == rank) return;
      const char *src = static_cast<const char *>(A_peers[o]) + static_cast<size_t>(r0) * pitch;
      char *dst = static_cast<char *>(A) + static_cast<size_t>(r0) * pitch;
      if (cudaMemcpy2DAsync(dst, pitch, src, pitch, static_cast<size_t>(k) * 2, static_cast<size_t>(r1 - r0),
                            cudaMemcpyDeviceToDevice, stream) != cudaSuccess)
        st = HGEMM_ERR_CUDA;
    });
  }
  if (st != HGEMM_SUCCESS) return st;
  return hgemm_core(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, 'T', transB, out_dtype, stream, nullptr);
}

hgemm_status_t hgemm_ipc_get_handle(const void *dptr, hgemm_ipc_handle_t *out) {
  if (!dptr || !out) return HGEMM_ERR_INVALID_VALUE;
  static MemGetAddressRangeFn range = driver_fn<MemGetAddressRangeFn>("cuMemGetAddressRange");
  if (!range) return HGEMM_ERR_CUDA;
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, reinterpret_cast<CUdeviceptr>(dptr)) != CUDA_SUCCESS) return HGEMM_ERR_INVALID_VALUE;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, reinterpret_cast<void *>(base)) != cudaSuccess) return HGEMM_ERR_CUDA;
  static_assert(sizeof(h) == sizeof(out->handle), "cudaIpcMemHandle_t size");
  std::memcpy(out->handle, &h, sizeof(h));
  out->offset = static_cast<int64_t>(reinterpret_cast<CUdeviceptr>(dptr) - base);
  return HGEMM_SUCCESS;
}

hgemm_status_t hgemm_ipc_open(const hgemm_ipc_handle_t *h, void **dptr) {
  if (!h || !dptr || h->offset < 0) return HGEMM_ERR_INVALID_VALUE;
  cudaIpcMemHandle_t ch;
  std::memcpy(&ch, h->handle, sizeof(ch));
  void *base = nullptr;
  if (cudaIpcOpenMemHandle(&base, ch, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) return HGEMM_ERR_CUDA;
  void *user = static_cast<char *>(base) + h->offset;
  std::lock_guard<std::mutex> lk(g_ipc_mu);
  if (g_ipc_n == static_cast<int>(sizeof(g_ipc) / sizeof(g_ipc[0]))) {
    cudaIpcCloseMemHandle(base);
    return HGEMM_ERR_CUDA;
  }
  g_ipc[g_ipc_n++] = {user, base};
  *dptr = user;
  return HGEMM_SUCCESS;
}

hgemm_status_t hgemm_ipc_close(void *dptr) {
  if (!dptr) return HGEMM_ERR_INVALID_VALUE;
  void *base = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_ipc_mu);
    for (int i = 0; i < g_ipc_n; ++i)
      if (g_ipc[i].user == dptr) {
        base = g_ipc[i].base;
        g_ipc[i] = g_ipc[--g_ipc_n];
        break;
      }
  }
  if (!base) return HGEMM_ERR_INVALID_VALUE;
  return cudaIpcCloseMemHandle(base) == cudaSuccess ? HGEMM_SUCCESS : HGEMM_ERR_CUDA;
}

}  // extern "C"
