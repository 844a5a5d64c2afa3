// curve_toy_a2.cu -- instantiation of the MSM pipeline for TOY_A2 (one TU per curve so
// the curves compile in parallel).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_toy_a2() { return Impl<TOY_A2>::get(); }
}  // namespace gzkp
