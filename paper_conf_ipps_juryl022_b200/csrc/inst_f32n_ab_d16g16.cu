// Explicit instantiations of the fused diagonal kernel (split across translation units
// so the template variants compile in parallel; see build.py).
#define MP_DIAG_IMPL
#include "mp_diag.cuh"
namespace mpk {
template struct Inst<float, 16, 16, 1, false, false>;
}  // namespace mpk
