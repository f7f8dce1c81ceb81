// Instantiations of the persistent tile kernel, CTA pair (cta_group::2), 256 x 256 pair tile
// (double-buffered accumulators): all layouts, the fused all-gather variants and the
// FP16-accumulate variants.
#include "hgemm_internal.cuh"

namespace hgi {

hgemm_status_t dispatch_tc256x2(int mc, bool ag, bool acc16, bool a_mn, bool b_mn, bool f32, const TcLaunch &L,
                                bool direct) {
#ifdef HGEMM_ENABLE_MC
  if (mc == 2) return dispatch_tc_layout<256, 2, 2>(a_mn, b_mn, f32, L);
#endif
  (void)mc;
  if (ag) return dispatch_tc_ag<256>(a_mn, f32, L);
  if (acc16) return f32 ? HGEMM_ERR_INVALID_VALUE : dispatch_tc_acc16<256>(a_mn, b_mn, L);
  // The direct-store epilogue variant (TcShape EPI_DIRECT: one more ring stage, 7 x 32 KB,
  // instead of the staging boxes) measured slower on every shape (profiles/r02/
  // epi_direct_experiment.log); it is instantiated only in experiment builds.
#ifdef HGEMM_ENABLE_EPI_DIRECT
  if (direct) return dispatch_tc_layout<256, 2, 1, true>(a_mn, b_mn, f32, L);
#else
  (void)direct;
#endif
  return dispatch_tc_layout<256, 2, 1>(a_mn, b_mn, f32, L);
}

hgemm_status_t dispatch_tc256_kg2(int cg, bool f32, const TcLaunch &L, int mc) {
  // 1-SM 128 x 128 tiles: three 64 KB stages, like the CTA-pair 256-wide tile (the 1-SM
  // 256-wide tile would have two 96 KB stages only: not built)
  if (cg == 1) return f32 ? launch_tc<128, 1, false, false, true, 1, false, false, false, 2>(L)
                          : launch_tc<128, 1, false, false, false, 1, false, false, false, 2>(L);
#ifdef HGEMM_ENABLE_MC
  if (mc == 2)
    return f32 ? launch_tc<256, 2, false, false, true, 2, false, false, false, 2>(L)
               : launch_tc<256, 2, false, false, false, 2, false, false, false, 2>(L);
#else
  (void)mc;
#endif
  return f32 ? launch_tc<256, 2, false, false, true, 1, false, false, false, 2>(L)
             : launch_tc<256, 2, false, false, false, 1, false, false, false, 2>(L);
}

}  // namespace hgi
