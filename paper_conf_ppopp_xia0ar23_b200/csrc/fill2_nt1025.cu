// fill2 kernels instantiated for 1024-thread CTAs with the one-CTA-per-SM register budget
// (kernel key 1025, see NtCfg in fill2_impl.cuh).
#include "fill2_impl.cuh"

namespace lusym {
LUSYM_F2_INSTANTIATE(1025)
}  // namespace lusym
