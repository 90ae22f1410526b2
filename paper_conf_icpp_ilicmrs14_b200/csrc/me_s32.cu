// me_s32.cu -- ME kernel instantiations for the compile-time window size S = 32
// (SA 32 x 32); see launch.cuh.
#include "launch.cuh"

namespace feves {
FEVES_ME_TU_DEF(32)
}  // namespace feves
