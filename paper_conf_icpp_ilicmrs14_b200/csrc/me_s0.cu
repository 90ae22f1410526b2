// me_s0.cu -- ME kernel instantiations for the compile-time window size S = 0
// (0 = run-time S: other even sizes, the inclusive SA, S = 128 with a predictor); see launch.cuh.
#include "launch.cuh"

namespace feves {
FEVES_ME_TU_DEF(0)
}  // namespace feves
