// sme_satd.cu -- SME kernel instantiations with the Hadamard SATD distortion (G20, f4).
#include "launch.cuh"

namespace feves {
cudaError_t sme_launch_satd(bool rd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P) {
  if (rd) sme_refine_kernel<true, true><<<grid, threads, 0, st>>>(P);
  else sme_refine_kernel<false, true><<<grid, threads, 0, st>>>(P);
  return cudaGetLastError();
}
}  // namespace feves
