// sme.cu -- SME kernel instantiations with SAD distortion (sme_refine.cuh); see launch.cuh.
// The Hadamard (SATD, G20) instantiations are in sme_satd.cu (compiled in parallel).
#include "launch.cuh"
#include "sme_smem.cuh"

namespace feves {
cudaError_t sme_launch_satd(bool rd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P);

cudaError_t sme_launch(bool rd, bool satd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P) {
  if (satd) return sme_launch_satd(rd, grid, threads, st, P);
  if (rd) sme_refine_kernel<true, false><<<grid, threads, 0, st>>>(P);
  else sme_refine_kernel<false, false><<<grid, threads, 0, st>>>(P);
  return cudaGetLastError();
}
cudaError_t sme2_init() {
  cudaError_t e = cudaFuncSetAttribute(sme_smem_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSme2Smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sme_smem_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSme2Smem);
  return e;
}

cudaError_t sme2_launch(bool rd, int n_units, cudaStream_t st, const SmeParams& P, int* ovf) {
  const int n_groups = n_units;   // groups of kSme2Mb MBs x rows x RFs
  cudaError_t e = cudaMemsetAsync(ovf, 0, sizeof(int), st);
  if (e != cudaSuccess) return e;
  const dim3 g2(2 * 148, 7);
  if (rd) {
    sme_smem_kernel<true><<<n_groups, kSme2Threads, kSme2Smem, st>>>(P, ovf);
    sme_list_kernel<true><<<g2, 128, 0, st>>>(P, ovf);
  } else {
    sme_smem_kernel<false><<<n_groups, kSme2Threads, kSme2Smem, st>>>(P, ovf);
    sme_list_kernel<false><<<g2, 128, 0, st>>>(P, ovf);
  }
  return cudaGetLastError();
}
}  // namespace feves
