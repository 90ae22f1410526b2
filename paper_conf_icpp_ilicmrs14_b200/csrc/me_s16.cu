// me_s16.cu -- ME kernel instantiations for the compile-time window size S = 16
// (SA 16 x 16); see launch.cuh.
#include "launch.cuh"

namespace feves {
FEVES_ME_TU_DEF(16)
}  // namespace feves
