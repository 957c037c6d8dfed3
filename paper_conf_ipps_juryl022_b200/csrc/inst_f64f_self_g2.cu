// Explicit instantiations of the FP64 fused kernel with the FP32 filter.
#define MP_DIAG_IMPL
#include "mp_diag64f.cuh"
namespace mpk {
template struct Inst64F<16, 2, true>;
}  // namespace mpk
