// Explicit instantiations of the block-cooperative large-d half kernel (parallel build, see build.py).
#define MP_DIAG_IMPL
#include "mp_diag_cta16.cuh"
namespace mpk {
#if MP_CTAH_NW
template struct InstCtaH<8, 8, CtaShapeH<8>::NW, false, 3>;
#endif
}  // namespace mpk
