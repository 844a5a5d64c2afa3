// curve_mnt4_753.cu -- instantiation of the MSM pipeline for MNT4_753 (one TU per curve so
// the curves compile in parallel).
#include "curves.cuh"
#include "msm_host.cuh"

namespace gzkp {
const CurveImpl* impl_mnt4_753() { return Impl<MNT4_753>::get(); }
}  // namespace gzkp
