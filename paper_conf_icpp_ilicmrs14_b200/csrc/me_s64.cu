// me_s64.cu -- ME kernel instantiations for the compile-time window size S = 64
// (SA 64 x 64); see launch.cuh.
#include "launch.cuh"
#include "me_ws.cuh"

namespace feves {
FEVES_ME_TU_DEF(64)

size_t me_ws_smem_bytes_64() { return (size_t)me_ws_smem_words() * 4; }
cudaError_t me_ws_init_64() {
  return cudaFuncSetAttribute(me_ws_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)me_ws_smem_bytes_64());
}
// persistent grid: resident CTAs per SM x SMs (queried once per device), at most one CTA per MB
cudaError_t me_ws_launch_64(dim3 grid, cudaStream_t st, const MeParams& P) {
  static int resident[64] = {0};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  if (!resident[dev]) {
    int sms = 0, per_sm = 0;
    if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess ||
        (e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, me_ws_kernel, kWsThreads, me_ws_smem_bytes_64())) !=
            cudaSuccess)
      return e;
    resident[dev] = std::max(1, sms * per_sm);
  }
  const int n_mb = (int)(grid.x * grid.y);
  me_ws_kernel<<<std::min(n_mb, resident[dev]), kWsThreads, me_ws_smem_bytes_64(), st>>>(P, n_mb);
  return cudaGetLastError();
}
}  // namespace feves
