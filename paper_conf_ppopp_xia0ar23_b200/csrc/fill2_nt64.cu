// fill2 kernels instantiated for 64-thread CTAs (see fill2_impl.cuh).
#include "fill2_impl.cuh"

namespace lusym {
LUSYM_F2_INSTANTIATE(64)
}  // namespace lusym
