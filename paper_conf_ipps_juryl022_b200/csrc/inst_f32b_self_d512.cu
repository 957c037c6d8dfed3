// Explicit instantiations of the fused diagonal kernel (split across translation units
// so the template variants compile in parallel; see build.py).
#define MP_DIAG_IMPL
#include "mp_diag_ctab.cuh"
namespace mpk {
template struct InstCtab<ctab_dl(512), 512 / ctab_dl(512), MP_CTAB_NT, true>;
}  // namespace mpk
