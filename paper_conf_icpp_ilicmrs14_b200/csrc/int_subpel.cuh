// int_subpel.cuh -- INT: the 16 quarter-pel phase planes of one RF.
//
// P:6: "the RFs are interpolated by applying 6tap and linear filters in the
// Interpolation (INT). The output of the INT is stored in a Sub-pixel
// interpolated Frame (SF) structure, which size is as large as 16 RFs."
// Filter (O2, the H.264 luma interpolation the paper inherits via
// JM 18.4): tap (1,-5,20,20,-5,1); b,h,m,s = Clip1((x1+16)>>5);
// j = Clip1((j1+512)>>10) with j1 taken horizontally over h1 (equal to the
// vertical form, pin P6); the 12 quarter samples are (u+v+1)>>1 averages,
// done four at a time with VAVRG4.
//
// One thread = 16 consecutive plane columns of one plane row; a warp writes
// 32 x 16 B = 512 contiguous bytes per plane with 128-bit stores (HBM-bound
// kernel: 1 B read + 16 B written per position).
#pragma once
#include "common.cuh"

namespace feves {

struct IntParams {
  const uint8_t* rf;
  uint8_t* sf;
  int W, H, pad, pitch, rows, row_begin, row_end;
  size_t plane;   // bytes per phase plane = rows * pitch
};

__device__ __forceinline__ int tap6(int a, int b, int c, int d, int e, int f) {
  return (a + f) - 5 * (b + e) + 20 * (c + d);
}
__device__ __forceinline__ uint32_t clip255(int v) { return (uint32_t)min(max(v, 0), 255); }

__device__ __forceinline__ uint32_t pack4(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  return __byte_perm(__byte_perm(a, b, 0x0040), __byte_perm(c, d, 0x0040), 0x5410);
}

__global__ void __launch_bounds__(128) int_subpel_kernel(const IntParams P) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;    // 16-column group
  const int rr = P.row_begin + blockIdx.y * blockDim.y + threadIdx.y;
  if (16 * g >= P.pitch || rr >= P.row_end) return;
  const int x0 = 16 * g - P.pad, y = rr - P.pad;

  // source rows y-2 .. y+3, columns x0-4 .. x0+19 (6 words per row)
  uint32_t w[6][6];
#pragma unroll
  for (int k = 0; k < 6; ++k)
#pragma unroll
    for (int q = 0; q < 6; ++q) w[k][q] = load4_clamped(P.rf, P.W, P.H, x0 - 4 + 4 * q, y - 2 + k);
  auto px = [&](int k, int c) -> int { return (int)((w[k][c >> 2] >> (8 * (c & 3))) & 0xffu); };  // c: col - (x0-4)

  // h1 at columns x0-2 .. x0+18 (index j <-> column x0-2+j), vertical taps
  int h1[21];
#pragma unroll
  for (int j = 0; j < 21; ++j)
    h1[j] = tap6(px(0, j + 2), px(1, j + 2), px(2, j + 2), px(3, j + 2), px(4, j + 2), px(5, j + 2));

  uint32_t Gw[4], Hw[4], Mw[4], bw[4], hw[4], mw[4], sw[4], jw[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint32_t G[4], Hh[4], M[4], b[4], h[4], m[4], s[4], j[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int i = 4 * q + u;                 // position x0 + i; row-2 column index i+4
      G[u] = px(2, i + 4);
      Hh[u] = px(2, i + 5);
      M[u] = px(3, i + 4);
      const int b1 = tap6(px(2, i + 2), px(2, i + 3), px(2, i + 4), px(2, i + 5), px(2, i + 6), px(2, i + 7));
      const int s1 = tap6(px(3, i + 2), px(3, i + 3), px(3, i + 4), px(3, i + 5), px(3, i + 6), px(3, i + 7));
      const int j1 = tap6(h1[i], h1[i + 1], h1[i + 2], h1[i + 3], h1[i + 4], h1[i + 5]);
      b[u] = clip255((b1 + 16) >> 5);
      s[u] = clip255((s1 + 16) >> 5);
      h[u] = clip255((h1[i + 2] + 16) >> 5);
      m[u] = clip255((h1[i + 3] + 16) >> 5);
      j[u] = clip255((j1 + 512) >> 10);
    }
    Gw[q] = pack4(G[0], G[1], G[2], G[3]);
    Hw[q] = pack4(Hh[0], Hh[1], Hh[2], Hh[3]);
    Mw[q] = pack4(M[0], M[1], M[2], M[3]);
    bw[q] = pack4(b[0], b[1], b[2], b[3]);
    hw[q] = pack4(h[0], h[1], h[2], h[3]);
    mw[q] = pack4(m[0], m[1], m[2], m[3]);
    sw[q] = pack4(s[0], s[1], s[2], s[3]);
    jw[q] = pack4(j[0], j[1], j[2], j[3]);
  }

  uint8_t* dst = P.sf + (size_t)rr * P.pitch + 16 * g;
  auto put = [&](int ph, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    *reinterpret_cast<uint4*>(dst + ph * P.plane) = make_uint4(a, b, c, d);
  };
#define PLANE(ph, EXPR) put(ph, EXPR(0), EXPR(1), EXPR(2), EXPR(3))
#define G_(q) Gw[q]
#define A_(q) vavg4(Gw[q], bw[q])
#define B_(q) bw[q]
#define C_(q) vavg4(Hw[q], bw[q])
#define D_(q) vavg4(Gw[q], hw[q])
#define E_(q) vavg4(bw[q], hw[q])
#define F_(q) vavg4(bw[q], jw[q])
#define Gq_(q) vavg4(bw[q], mw[q])
#define H_(q) hw[q]
#define I_(q) vavg4(hw[q], jw[q])
#define J_(q) jw[q]
#define K_(q) vavg4(jw[q], mw[q])
#define N_(q) vavg4(Mw[q], hw[q])
#define Pq_(q) vavg4(hw[q], sw[q])
#define Q_(q) vavg4(jw[q], sw[q])
#define R_(q) vavg4(mw[q], sw[q])
  // phase = 4*yFrac + xFrac (G11); names as in DESIGN.md O2
  PLANE(0, G_);  PLANE(1, A_);  PLANE(2, B_);   PLANE(3, C_);
  PLANE(4, D_);  PLANE(5, E_);  PLANE(6, F_);   PLANE(7, Gq_);
  PLANE(8, H_);  PLANE(9, I_);  PLANE(10, J_);  PLANE(11, K_);
  PLANE(12, N_); PLANE(13, Pq_); PLANE(14, Q_); PLANE(15, R_);
#undef PLANE
#undef G_
#undef A_
#undef B_
#undef C_
#undef D_
#undef E_
#undef F_
#undef Gq_
#undef H_
#undef I_
#undef J_
#undef K_
#undef N_
#undef Pq_
#undef Q_
#undef R_
}

}  // namespace feves
