// common.cuh -- small device helpers shared by the sm_100a kernels of
// libfeves_me.so.  (Product code: never shared with oracle/.)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace feves {

constexpr int kNPart = 41;     // partitions of the 7 modes (P:6), order G7
constexpr int kMaxRf = 16;

// d = c + sum_{i<4} |a.byte_i - b.byte_i|  -> one VABSDIFF4.U8.ACC (SURVEY §2.7,
// verified in SASS; the intrinsic __vsadu4 does not chain the accumulator).
__device__ __forceinline__ uint32_t vad4(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("vabsdiff4.u32.u32.u32.add %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

// per-byte rounded average (u+v+1)>>1 on 4 packed bytes.  PTX vavrg4 is NOT
// native on sm_100a (ptxas expands it byte by byte, ~16 instructions).  Exact
// SWAR form: ceil((a+b)/2) = y + (x >> 1) per byte with
//   y = (a & b) | ((a ^ b) & 0x01)   (= floor part + carry-in bit; ONE LOP3),
//   x = (a ^ b) & 0xfe               (ONE LOP3; bit 0 of every byte cleared, so
//                                     the 32-bit shift moves nothing across bytes),
// and y + (x >> 1) = hi32(x * 2^31) + y as ONE IMAD.HI on the FMA pipe (the
// per-byte sum is the average <= 255, so no carry crosses a byte).  k_hi must be
// 0x80000000 supplied at run time (a kernel parameter): a literal would be
// strength-reduced by ptxas into SHF + IADD on the ALU pipe, which is the pipe
// INT and SME are bound by.  2 ALU + 1 FMA instead of 4 ALU + 1 FMA.
// (Checked exhaustively over all byte pairs on the host; parity tests.)
__device__ __forceinline__ uint32_t vavg4(uint32_t a, uint32_t b, uint32_t k_hi) {
  const uint32_t y = (a & b) | ((a ^ b) & 0x01010101u);
  const uint32_t x = (a ^ b) & 0xfefefefeu;
  uint32_t d;
  asm("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(x), "r"(k_hi), "r"(y));
  return d;
}
constexpr uint32_t kAvgHi = 0x80000000u;   // the run-time k_hi of vavg4 (host side)

__device__ __forceinline__ int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

// Four bytes of row y of a W x H tight u8 frame starting at column x, with
// coordinate clamping (G5).  Fast paths: one aligned 32-bit load inside the
// frame; one byte load broadcast when the 4 columns all clamp to the same edge.
__device__ __forceinline__ uint32_t load4_clamped(const uint8_t* __restrict__ f, int W, int H, int x, int y) {
  y = clampi(y, 0, H - 1);
  const uint8_t* row = f + (size_t)y * W;
  if (x >= 0 && x + 3 < W && ((reinterpret_cast<uintptr_t>(row + x) & 3) == 0))
    return __ldg(reinterpret_cast<const uint32_t*>(row + x));
  if (x + 3 <= 0) return 0x01010101u * __ldg(row);
  if (x >= W - 1) return 0x01010101u * __ldg(row + W - 1);
  uint32_t v = 0;
#pragma unroll
  for (int i = 0; i < 4; ++i) v |= (uint32_t)__ldg(row + clampi(x + i, 0, W - 1)) << (8 * i);
  return v;
}

}  // namespace feves
