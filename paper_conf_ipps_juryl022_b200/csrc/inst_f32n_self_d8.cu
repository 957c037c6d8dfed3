// Explicit instantiations of the fused diagonal kernel (split across translation units
// so the template variants compile in parallel; see build.py).
#define MP_DIAG_IMPL
#include "mp_diag.cuh"
namespace mpk {
template struct Inst<float, 8, 1, 2, true, false>;
}  // namespace mpk
