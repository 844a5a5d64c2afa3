// curve_toy_a0.cu -- instantiation of the MSM pipeline for TOY_A0 (one TU per curve so
// the curves compile in parallel).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_toy_a0() { return Impl<TOY_A0>::get(); }
}  // namespace gzkp
