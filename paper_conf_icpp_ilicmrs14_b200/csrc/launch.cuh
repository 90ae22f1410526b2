// launch.cuh -- host-side launch entry points of the kernels, one translation unit
// per ME window size (me_s*.cu) and one for SME (sme.cu), so the many template
// instantiations compile in parallel.  feves_me.cu (the C-ABI) calls only these.
#pragma once
#include <algorithm>
#include "me_fsbm.cuh"
#include "sme_refine.cuh"

namespace feves {

// ME kernel variants (template arguments of me_fsbm_kernel)
enum MeVariant : int {
  kMePlain = 0,     // pure SAD (G3)
  kMeFused = 1,     // + SME of the CTA's own MB (ME_OPT_FUSED_SME)
  kMeRate = 2,      // J = SAD + lambda * R (G18), key shift 15
  kMePmv = 3,       // predicted-MV centre (G21)
  kMePmvRate = 4,   // both
};

template <int SS>
inline cudaError_t me_launch_tmpl(int variant, dim3 grid, int threads, size_t smem, cudaStream_t st,
                                  const MeParams& P) {
  switch (variant) {
    case kMeFused: me_fsbm_kernel<SS, true><<<grid, threads, smem, st>>>(P); break;
    case kMeRate: me_fsbm_kernel<SS, false, 15><<<grid, threads, smem, st>>>(P); break;
    case kMePmv:
      if constexpr (SS != 128) { me_fsbm_kernel<SS, false, 16, true><<<grid, threads, smem, st>>>(P); break; }
      return cudaErrorInvalidValue;   // S = 128 with a predictor runs the runtime-S kernel (SS = 0)
    case kMePmvRate:
      if constexpr (SS != 128) { me_fsbm_kernel<SS, false, 15, true><<<grid, threads, smem, st>>>(P); break; }
      return cudaErrorInvalidValue;
    default: me_fsbm_kernel<SS, false><<<grid, threads, smem, st>>>(P); break;
  }
  return cudaGetLastError();
}

template <int SS>
inline cudaError_t me_set_smem_tmpl(int bytes) {
  cudaError_t e = cudaFuncSetAttribute(me_fsbm_kernel<SS>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(me_fsbm_kernel<SS, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(me_fsbm_kernel<SS, false, 15>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if constexpr (SS != 128) {
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(me_fsbm_kernel<SS, false, 16, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(me_fsbm_kernel<SS, false, 15, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  }
  return e;
}

#define FEVES_ME_TU_DECL(SS)                                                                          \
  cudaError_t me_launch_##SS(int variant, dim3 grid, int threads, size_t smem, cudaStream_t st,      \
                             const MeParams& P);                                                      \
  cudaError_t me_set_smem_##SS(int bytes);
FEVES_ME_TU_DECL(0)
FEVES_ME_TU_DECL(16)
FEVES_ME_TU_DECL(32)
FEVES_ME_TU_DECL(64)
FEVES_ME_TU_DECL(128)
#undef FEVES_ME_TU_DECL

#define FEVES_ME_TU_DEF(SS)                                                                           \
  cudaError_t me_launch_##SS(int variant, dim3 grid, int threads, size_t smem, cudaStream_t st,      \
                             const MeParams& P) {                                                     \
    return me_launch_tmpl<SS>(variant, grid, threads, smem, st, P);                                   \
  }                                                                                                   \
  cudaError_t me_set_smem_##SS(int bytes) { return me_set_smem_tmpl<SS>(bytes); }

// SME (sme.cu): rd = rate term compiled in (G18), satd = Hadamard distortion (G20)
cudaError_t sme_launch(bool rd, bool satd, dim3 grid, int threads, cudaStream_t st, const SmeParams& P);
// SME with shared-memory staged windows (sme_smem.cuh), one CTA per group of 8 MBs x RF:
// ovf = device int[1 + n_groups] overflow list (counter reset here), then the global-load
// kernel on the overflow groups
cudaError_t sme2_launch(bool rd, int n_groups, cudaStream_t st, const SmeParams& P, int* ovf);
cudaError_t sme2_init();   // dynamic shared-memory attribute (once per process/device)

}  // namespace feves
