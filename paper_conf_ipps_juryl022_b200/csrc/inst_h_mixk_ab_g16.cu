// Explicit instantiations of the half2 fused diagonal kernel (FP16 / Mixed / FP16C).
#define MP_DIAG_IMPL
#include "mp_diag16.cuh"
namespace mpk {
template struct InstH<8, 16, false, 3>;
}  // namespace mpk
