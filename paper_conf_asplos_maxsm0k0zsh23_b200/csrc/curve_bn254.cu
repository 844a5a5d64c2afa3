// curve_bn254.cu -- instantiation of the MSM pipeline for BN254 (one TU per curve so
// the curves compile in parallel).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_bn254() { return Impl<BN254>::get(); }
}  // namespace gzkp
