// curve_bls12_381_g2.cu -- the MSM pipeline instantiated for BLS12-381 G2 (F_p^2
// coordinates).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_bls12_381_g2() { return Impl<BLS12_381_G2>::get(); }
}  // namespace gzkp
