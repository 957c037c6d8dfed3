// Explicit instantiations of the block-cooperative large-d FP32 kernel (parallel build, see build.py).
#define MP_DIAG_IMPL
#include "mp_diag_cta.cuh"
namespace mpk {
#if MP_CTA_NW && MP_CTA_MIN_DP < 64
template struct InstCta<16, 2, MP_CTA_NW, false>;
#endif
}  // namespace mpk
