// me_s64.cu -- ME kernel instantiations for the compile-time window size S = 64
// (SA 64 x 64); see launch.cuh.
#include "launch.cuh"

namespace feves {
FEVES_ME_TU_DEF(64)
}  // namespace feves
