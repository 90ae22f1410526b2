// me_s128.cu -- ME kernel instantiations for the compile-time window size S = 128
// (SA 128 x 128); see launch.cuh.
#include "launch.cuh"

namespace feves {
FEVES_ME_TU_DEF(128)
}  // namespace feves
