// L1 cost model of the SME's gather loads (SME): how many L1TEX data-pipe
// wavefronts does one warp-wide global load cost for the access patterns the SME kernel
// can produce?  Each pattern kernel issues ITERS loads per warp over an L2-resident buffer;
// run under ncu with l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum and
// smsp__inst_executed_op_global_ld.sum and divide.
//   p0 LDG.32  32 lanes, one aligned 128-B line                (coalesced reference)
//   p1 LDG.32  8 groups x 4 lanes, 16 B each, 8 distinct lines (SME, MVs differ per MB)
//   p2 LDG.32  as p1, groups start 4 bytes before a line end     (segment crosses a line)
//   p3 LDG.64  8 groups x 4 lanes, 8 B each (32 B per group)
//   p4 LDG.128 8 groups x 4 lanes, all 4 lanes of a group the same 16 B
//   p5 LDG.128 8 groups x 4 lanes, 16 B each (64 B per group)
//   p6 LDG.32  16 groups x 2 lanes, 16 distinct lines
//   p7 LDG.32  32 lanes, 32 distinct lines
//   p8 LDG.32 x 2 per iteration (words w, w+1; 8 groups x 4 lanes, 8 lines)  -- the SME's window row
//   p9 LDG.32 + TLD (tex1Dfetch) for w+1: does the texture path add L1 throughput beside the LSU?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int ITERS = 512;

template <int P>
__global__ void __launch_bounds__(256) gather(const uint8_t* __restrict__ buf, uint32_t* out, int stride,
                                              cudaTextureObject_t tex) {
  const int lane = threadIdx.x & 31, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int g = lane >> 2, q = lane & 3;
  uint32_t acc = 0;
  size_t base = (size_t)(warp & 1023) * 64 * 1024;
  for (int it = 0; it < ITERS; ++it) {
    const size_t row = base + (size_t)((it * 37) & 255) * stride;   // a new row each load
    if (P == 0) acc += *reinterpret_cast<const uint32_t*>(buf + row + 4 * lane);
    if (P == 1) acc += __ldg(reinterpret_cast<const uint32_t*>(buf + row + 2048 * g + 4 * q));
    if (P == 2) acc += __ldg(reinterpret_cast<const uint32_t*>(buf + row + 2048 * g + 124 + 4 * q));
    if (P == 3) { const uint2 v = __ldg(reinterpret_cast<const uint2*>(buf + row + 2048 * g + 8 * q)); acc += v.x ^ v.y; }
    if (P == 4) { const uint4 v = __ldg(reinterpret_cast<const uint4*>(buf + row + 2048 * g)); acc += v.x ^ v.y ^ v.z ^ v.w; }
    if (P == 5) { const uint4 v = __ldg(reinterpret_cast<const uint4*>(buf + row + 2048 * g + 16 * q)); acc += v.x ^ v.y ^ v.z ^ v.w; }
    if (P == 6) acc += __ldg(reinterpret_cast<const uint32_t*>(buf + row + 2048 * (lane >> 1) + 4 * (lane & 1)));
    if (P == 7) acc += __ldg(reinterpret_cast<const uint32_t*>(buf + row + 2048 * lane));
    if (P == 8) {
      const uint32_t* p = reinterpret_cast<const uint32_t*>(buf + row + 2048 * g + 4 * q);
      acc += __funnelshift_r(__ldg(p), __ldg(p + 1), acc & 24);
    }
    if (P == 9) {
      const size_t wi = (row + 2048 * g + 4 * q) >> 2;
      acc += __funnelshift_r(__ldg(reinterpret_cast<const uint32_t*>(buf) + wi), tex1Dfetch<uint32_t>(tex, (int)(wi + 1)),
                             acc & 24);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
  const size_t bytes = 96ull << 20;   // L2-resident (126 MB L2)
  uint8_t* buf; uint32_t* out;
  cudaMalloc(&buf, bytes); cudaMemset(buf, 1, bytes);
  const int blocks = 148 * 4, thr = 256;
  cudaMalloc(&out, 4 * blocks * thr);
  const int stride = 2016 * 0 + 64 * 1024 / 256;   // rows inside the warp's 64 KB slab
  cudaResourceDesc rd = {};
  rd.resType = cudaResourceTypeLinear;
  rd.res.linear.devPtr = buf;
  rd.res.linear.desc = cudaCreateChannelDesc<uint32_t>();
  rd.res.linear.sizeInBytes = bytes;
  cudaTextureDesc td = {};
  td.readMode = cudaReadModeElementType;
  cudaTextureObject_t tex = 0;
  if (cudaCreateTextureObject(&tex, &rd, &td, nullptr) != cudaSuccess) { printf("texture object failed\n"); return 1; }
  float ms;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
#define RUN(P)                                                            \
  gather<P><<<blocks, thr>>>(buf, out, stride, tex);                       \
  cudaEventRecord(a); gather<P><<<blocks, thr>>>(buf, out, stride, tex); cudaEventRecord(b); \
  cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);               \
  printf("p%d: %.3f us per launch, %.2f ns per warp-load per SM\n", P, ms * 1e3, ms * 1e6 / (blocks * thr / 32 * ITERS / 148.0));
  RUN(0) RUN(1) RUN(2) RUN(3) RUN(4) RUN(5) RUN(6) RUN(7) RUN(8) RUN(9)
  return 0;
}
