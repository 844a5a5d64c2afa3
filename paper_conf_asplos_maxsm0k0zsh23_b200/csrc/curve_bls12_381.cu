// curve_bls12_381.cu -- instantiation of the MSM pipeline for BLS12_381 (one TU per curve so
// the curves compile in parallel).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_bls12_381() { return Impl<BLS12_381>::get(); }
}  // namespace gzkp
