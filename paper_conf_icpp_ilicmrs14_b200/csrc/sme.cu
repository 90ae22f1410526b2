// sme.cu -- SME kernel instantiations with SAD distortion (sme_refine.cuh); see launch.cuh.
// The Hadamard (SATD, G20) instantiations are in sme_satd.cu (compiled in parallel).
#include "launch.cuh"

namespace feves {
cudaError_t sme_launch_satd(bool rd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P);

cudaError_t sme_launch(bool rd, bool satd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P) {
  if (satd) return sme_launch_satd(rd, grid, threads, st, P);
  if (rd) sme_refine_kernel<true, false><<<grid, threads, 0, st>>>(P);
  else sme_refine_kernel<false, false><<<grid, threads, 0, st>>>(P);
  return cudaGetLastError();
}
}  // namespace feves
