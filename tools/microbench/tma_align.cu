// Does a 2-D TMA tile load (cp.async.bulk.tensor, SWIZZLE_NONE, u8) accept a shared-memory
// destination that is only 16- or 32-byte aligned, and a box start at any byte column?  (The ME
// window's 4 byte-shifted copies need an 8-word bank stagger between copies.)
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <cuda.h>
#include <cuda_runtime.h>

__global__ void tma_kernel(const __grid_constant__ CUtensorMap tmap, int x0, int y0, int dst_off, uint8_t* out) {
  __shared__ __align__(1024) uint8_t sm[16384];
  __shared__ __align__(8) uint64_t bar;
  const uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(sm) + dst_off;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(80 * 79) : "memory");
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(d), "l"(&tmap), "r"(x0), "r"(y0), "r"(b) : "memory");
  }
  asm volatile(
      "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(b) : "memory");
  for (int i = threadIdx.x; i < 80 * 79; i += blockDim.x) out[i] = sm[dst_off + i];
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int W = 1920, H = 1080;
  uint8_t* h = (uint8_t*)malloc(W * H);
  for (int i = 0; i < W * H; ++i) h[i] = (uint8_t)(i * 7 + (i / W) * 13);
  uint8_t *f, *o;
  cudaMalloc(&f, W * H); cudaMalloc(&o, 80 * 79);
  cudaMemcpy(f, h, W * H, cudaMemcpyHostToDevice);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {
    printf("no cuTensorMapEncodeTiled\n"); return 1;
  }
  CUtensorMap tm;
  cuuint64_t dims[2] = {(cuuint64_t)W, (cuuint64_t)H}, strides[1] = {(cuuint64_t)W};
  cuuint32_t box[2] = {80, 79}, es[2] = {1, 1};
  CUresult r = ((EncodeFn)fn)(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, f, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                              CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode: %d\n", (int)r);
  uint8_t* g = (uint8_t*)malloc(80 * 79);
  const int offs[] = {0, 16, 32, 96, 128, 160};
  const int xs[] = {64, 65, 66, 67};
  for (int off : offs)
    for (int x0 : xs) {
      tma_kernel<<<1, 128>>>(tm, x0, 100, off, o);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("dst_off %3d x0 %d: %s\n", off, x0, cudaGetErrorString(e)); return 0; }
      cudaMemcpy(g, o, 80 * 79, cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int yy = 0; yy < 79; ++yy)
        for (int xx = 0; xx < 80; ++xx) bad += g[yy * 80 + xx] != h[(100 + yy) * W + x0 + xx];
      printf("dst_off %3d x0 %d: %s\n", off, x0, bad ? "MISMATCH" : "ok");
    }
  return 0;
}
