// How busy can the ALU pipe get for the ME candidate loop's instruction mix?
// Per "candidate": 64 VABSDIFF4 (16 chains x 4) + 20 VIMNMX3 + 41 IMAD + 23 LDS, the
// per-candidate mix of me_fsbm_kernel<64>.  All asm volatile, so the
// order written is the order issued.  ORDER 0 = interleaved (every ALU op followed by a
// non-ALU op where the mix allows), 1 = bursty (all VABSDIFF4, then IMAD, VIMNMX3, LDS),
// 2 = the ME loop's shape (SAD runs, then key / fold bursts per block row).
// Output per (order, warps/SM): cycles per candidate-warp and the ALU-pipe busy fraction
// (2 cycles per ALU warp-instruction per SMSP).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t vad4(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d; asm volatile("vabsdiff4.u32.u32.u32.add %0,%1,%2,%3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ uint32_t mn3(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d; asm volatile("{.reg .u32 t; min.u32 t,%1,%2; min.u32 %0,t,%3;}" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ uint32_t mad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d; asm volatile("mad.lo.u32 %0,%1,%2,%3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ uint32_t lds(uint32_t a) {
  uint32_t d; asm volatile("ld.shared.u32 %0,[%1];" : "=r"(d) : "r"(a) : "memory"); return d; }

constexpr int ITERS = 256;

template <int ORDER>
__global__ void __launch_bounds__(128) kern(uint32_t seed, uint32_t* out, unsigned long long* cyc) {
  __shared__ uint32_t sm[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) sm[i] = i * seed;
  __syncthreads();
  uint32_t acc[16], M[20], K[8], C[8], W[4] = {1u, 2u, 3u, 4u};
#pragma unroll
  for (int i = 0; i < 16; ++i) acc[i] = seed * (i + 1) + threadIdx.x;
#pragma unroll
  for (int i = 0; i < 20; ++i) M[i] = 0xffffffffu - i;
#pragma unroll
  for (int i = 0; i < 8; ++i) { K[i] = seed ^ i; C[i] = seed * 3 + i * threadIdx.x; }
  uint32_t x = seed + threadIdx.x, y = seed * 7u, w = 0;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm) + 4 * (threadIdx.x & 31);
  __syncthreads();
  const unsigned long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
    if (ORDER == 0) {
      // 84 ALU ops (64 VABSDIFF4 + 20 VIMNMX3) with the 64 non-ALU ops (41 IMAD + 23 LDS)
      // spread evenly between them (Bresenham)
      int a = 0, m = 0, k = 0, l = 0;
#pragma unroll
      for (int j = 0; j < 84; ++j) {
        if (j % 4 == 3 && m < 20) { M[m] = mn3(M[m], K[m & 7], K[(m + 3) & 7]); ++m; }
        else if (a < 64) { acc[a & 15] = vad4(C[a & 7], W[a & 3], acc[a & 15]); ++a; }
        else { M[m % 20] = mn3(M[m % 20], K[m & 7], acc[m & 15]); ++m; }
        if ((j + 1) * 64 / 84 > j * 64 / 84) {
          if (l < 23 && (k + l) % 3 == 2) { W[l & 3] = lds(sbase + 128 * l); ++l; }
          else if (k < 41) { K[k & 7] = mad(acc[k & 15], 65536u, K[(k + 1) & 7]); ++k; }
          else { W[l & 3] = lds(sbase + 128 * l); ++l; }
        }
      }
    } else if (ORDER == 1) {
#pragma unroll
      for (int a = 0; a < 64; ++a) acc[a & 15] = vad4(C[a & 7], W[a & 3], acc[a & 15]);
#pragma unroll
      for (int k = 0; k < 41; ++k) K[k & 7] = mad(acc[k & 15], 65536u, K[(k + 1) & 7]);
#pragma unroll
      for (int m = 0; m < 20; ++m) M[m] = mn3(M[m], K[m & 7], K[(m + 3) & 7]);
#pragma unroll
      for (int l = 0; l < 23; ++l) W[l & 3] = lds(sbase + 128 * l);
    } else {
      // ME shape per 4 candidates scaled to 1: a row = 1 LDS.. 4 VABS; every 4 rows keys + folds
#pragma unroll
      for (int r = 0; r < 16; ++r) {
        W[r & 3] = lds(sbase + 128 * r);
#pragma unroll
        for (int b = 0; b < 4; ++b) acc[(r & 3) * 4 + b] = vad4(C[(r + b) & 7], W[b], acc[(r & 3) * 4 + b]);
        if ((r & 3) == 3) {
#pragma unroll
          for (int k = 0; k < 10; ++k) K[k & 7] = mad(acc[k & 15], 65536u, K[(k + 1) & 7]);
#pragma unroll
          for (int m = 0; m < 5; ++m) M[(r / 4) * 5 + m] = mn3(M[(r / 4) * 5 + m], K[m & 7], K[(m + 3) & 7]);
        }
      }
#pragma unroll
      for (int l = 0; l < 7; ++l) W[l & 3] = lds(sbase + 128 * (16 + l));
      K[0] = mad(acc[0], 65536u, K[1]);
    }
  }
  const unsigned long long t1 = clock64();
  uint32_t s = w + W[0] + W[1] + W[2] + W[3] + x + y;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += acc[i];
#pragma unroll
  for (int i = 0; i < 20; ++i) s ^= M[i];
#pragma unroll
  for (int i = 0; i < 8; ++i) s += K[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int O>
void run(int nsm, int warps) {
  uint32_t* out; unsigned long long* cyc;
  const int thr = 128, nb = nsm * (warps / 4);          // 4-warp CTAs, warps/4 per SM
  cudaMalloc(&out, 4 * nb * thr); cudaMalloc(&cyc, 8 * nb);
  kern<O><<<nb, thr>>>(1, out, cyc); cudaDeviceSynchronize();
  kern<O><<<nb, thr>>>(3, out, cyc); cudaDeviceSynchronize();
  static unsigned long long h[8192];
  cudaMemcpy(h, cyc, 8 * nb, cudaMemcpyDeviceToHost);
  double sum = 0; for (int i = 0; i < nb; ++i) sum += h[i];
  const double cyc_it = sum / nb / ITERS;                  // cycles per iteration (co-resident CTAs)
  const double per_smsp_warps = warps / 4.0;
  const double alu_cycles = 84.0 * 2 * per_smsp_warps;    // ALU cycles needed per iteration per SMSP
  const double issue = 148.0 * per_smsp_warps;
  printf("order %d warps/SM %2d: %7.1f cycles/iter  ALU busy %.3f  issue %.3f  -> px-roofline frac %.3f\n", O, warps,
         cyc_it, alu_cycles / cyc_it, issue / cyc_it, 64.0 * 2 * per_smsp_warps / cyc_it);
  cudaFree(out); cudaFree(cyc);
}

int main() {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  for (int w : {8, 12, 16, 20, 24}) { run<0>(nsm, w); run<1>(nsm, w); run<2>(nsm, w); }
  return 0;
}
