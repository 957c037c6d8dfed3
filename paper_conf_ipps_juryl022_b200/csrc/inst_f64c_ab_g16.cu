// Explicit instantiations of the block-cooperative large-d FP64 kernel (parallel build, see build.py).
#define MP_DIAG_IMPL
#include "mp_diag_cta64.cuh"
namespace mpk {
#if MP_CTA64_ON
template struct InstCta64<MP_CTA64_DL, 16, CtaShape64<16>::NW, false>;
#endif
}  // namespace mpk
