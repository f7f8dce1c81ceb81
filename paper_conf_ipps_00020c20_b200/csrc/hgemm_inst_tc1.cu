// Instantiations of the persistent tile kernel on one SM (cta_group::1): 128 x 256 and 128 x 128 tiles.
#include "hgemm_internal.cuh"

namespace hgi {

hgemm_status_t dispatch_tc1(int bn, bool a_mn, bool b_mn, bool f32, const TcLaunch &L) {
  if (bn == 256) return dispatch_tc_layout<256, 1, 1>(a_mn, b_mn, f32, L);
  return dispatch_tc_layout<128, 1, 1>(a_mn, b_mn, f32, L);
}

}  // namespace hgi
