// Instantiations of the split-K kernel (hgemm_splitk.cuh), 128 x 64 tiles, 2/4/8 splits, all layouts.
#include "hgemm_internal.cuh"

namespace hgi {

hgemm_status_t dispatch_splitk64(int spl, bool a_mn, bool b_mn, bool f32, const CUtensorMap &ta,
                                 const CUtensorMap &tb, const hg::TcParams &p, int dev, cudaStream_t s, bool hm) {
  // hm: 64 x 64 tiles (64 valid Ak rows, hgemm_splitk.cuh "HM"), 2 or 4 splits
  if (hm) {
    if (spl == 2) return dispatch_splitk_layout<64, 2, true>(a_mn, b_mn, f32, ta, tb, p, dev, s);
    if (spl == 4) return dispatch_splitk_layout<64, 4, true>(a_mn, b_mn, f32, ta, tb, p, dev, s);
    return HGEMM_ERR_INVALID_VALUE;
  }
  if (spl == 2) return dispatch_splitk_layout<64, 2>(a_mn, b_mn, f32, ta, tb, p, dev, s);
  if (spl == 4) return dispatch_splitk_layout<64, 4>(a_mn, b_mn, f32, ta, tb, p, dev, s);
  if (spl == 8) return dispatch_splitk_layout<64, 8>(a_mn, b_mn, f32, ta, tb, p, dev, s);
  return HGEMM_ERR_INVALID_VALUE;
}

}  // namespace hgi
