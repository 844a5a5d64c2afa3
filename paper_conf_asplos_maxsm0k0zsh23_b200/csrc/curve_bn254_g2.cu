// curve_bn254_g2.cu -- the MSM pipeline instantiated for BN254 G2 (F_p^2
// coordinates).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_bn254_g2() { return Impl<BN254_G2>::get(); }
}  // namespace gzkp
