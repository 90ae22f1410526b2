// int_subpel.cuh -- INT: the 16 quarter-pel phase planes of one RF.
//
// P:6: "the RFs are interpolated by applying 6tap and linear filters in the
// Interpolation (INT). The output of the INT is stored in a Sub-pixel
// interpolated Frame (SF) structure, which size is as large as 16 RFs."
// Filter (O2, the H.264 luma interpolation the paper inherits via
// JM 18.4): tap (1,-5,20,20,-5,1); b,h,m,s = Clip1((x1+16)>>5);
// j = Clip1((j1+512)>>10) with j1 taken horizontally over h1 (equal to the
// vertical form, pin P6); the 12 quarter samples are (u+v+1)>>1 averages.
//
// One thread = 16 consecutive plane columns of one plane row.  The 6-tap
// filters on b1/h1/s1 (range [-2550, 10710]) run two columns per 32-bit
// instruction on biased, non-negative 16-bit lanes (plain IADD / IMAD by 20
// and -5, exact per lane); j1 (20-bit) runs in int32.  Quarter samples: SWAR vavg4 on 4 packed
// bytes.  A warp writes 32 x 16 B = 512 contiguous bytes per plane with
// 128-bit stores (HBM-bound kernel: 1 B read + 16 B written per position).
#pragma once
#include "common.cuh"

namespace feves {

struct IntParams {
  const uint8_t* rf;
  uint8_t* sf;
  int W, H, pad, pitch, rows, row_begin, row_end;
  size_t plane;   // bytes per phase plane = rows * pitch
  int g_lo, g_hi; // interior 16-column groups [g_lo, g_hi): every source word in-frame and aligned
  int border_bx;  // border blocks: groups per block row (power of two >= number of border groups)
  uint32_t k_hi;  // = kAvgHi (vavg4)
  int vec_ok;     // W % 4 == 0 and rf 4-byte aligned: tile rows as aligned words (int_tile_kernel)
};

// Two columns per 32-bit register, one per 16-bit lane, and every lane kept
// NON-NEGATIVE so plain 32-bit IADD/IMAD are exact per lane (no carry or
// borrow can cross lanes).  A 6-tap result x1 in [-2550, 10710] is carried as
// x1 + B in [5658, 18918], B = 8208 = 256 * 32 + 16: the +16 is the rounding of
// (x1 + 16) >> 5, and 32 * B = 256 * 1024 + 512 is exactly the rounding of
// (j1 + 512) >> 10 plus 256 (j1 = the tap sum of six biased h1), so both
// shifted values come out as (rounded value) + 256 and the Clip1 to [0, 255] is
// a clamp to [256, 511] whose LOW BYTE is the sample -- no rounding add and no
// bias subtraction.  (No 16x2 subtraction: ptxas was seen to
// miscompile __vsub2 when one lane is dead.)
constexpr uint32_t kBias = 8208u;
constexpr uint32_t kBias2 = kBias | (kBias << 16);
// tap6 on packed byte columns: (a+f) - 5(b+e) + 20(c+d) + B, per lane
__device__ __forceinline__ uint32_t tap6x2b(uint32_t a, uint32_t b, uint32_t c, uint32_t d, uint32_t e, uint32_t f) {
  const uint32_t s = a + f, q = b + e, m = c + d;                   // lanes <= 510: no carry
  return (m * 20u + s) + (kBias2 - q * 5u);                          // lanes in [5658, 18918]
}
// Clip1((x1 + 16) >> 5) + 256 on two biased lanes: u16 lanes in [256, 511], low byte = sample
__device__ __forceinline__ uint32_t clip_half2(uint32_t vb) {
  const uint32_t t = (vb >> 5) & 0x07ff07ffu;                       // ((x1+16)>>5) + 256 per lane
  return __vminu2(__vmaxu2(t, 0x01000100u), 0x01ff01ffu);
}
__device__ __forceinline__ int lo_u16(uint32_t x) { return (int)(x & 0xffffu); }
__device__ __forceinline__ int hi_u16(uint32_t x) { return (int)(x >> 16); }
// Clip1((j1 + 512) >> 10) + 256 from the biased sum jb = j1 + 32 * B (> 0): low byte = j
__device__ __forceinline__ uint32_t clip_j(int jb) { return (uint32_t)min(max(jb >> 10, 256), 511); }

// low bytes of four u16 lanes (pairs a, b) -> one byte word
__device__ __forceinline__ uint32_t bytes_of(uint32_t a, uint32_t b) { return __byte_perm(a, b, 0x6420); }

// One launch, two kinds of blocks (uniform per block, so warps never diverge):
// blockIdx.z == 1: interior groups [g_lo, g_hi) with no clamping code at all;
// blockIdx.z == 0: the border groups, 128 threads = border_bx groups x rows per
// block, blockIdx.x = which border_bx-wide slice of the border groups (every
// border group is covered: all of them when W % 4 != 0 or the RF rows are not
// 4-byte aligned; dispatched first: they are the latency-bound tail otherwise).
// the 16 planes of 16 columns x 1 row (plane group g, plane row rr) from the source words
// w[k][q] = rows y-2 .. y+3 (k = 0..5), columns x0-4 .. x0+19 (q = 0..5), y = rr - pad, x0 = 16g - pad
__device__ __forceinline__ void int_compute(const IntParams& P, int g, int rr, const uint32_t (&w)[6][6]) {
  // byte pairs as u16x2: pr[k][j] = columns (2j, 2j+1)
  auto pr = [&](int k, int j) -> uint32_t { return __byte_perm(w[k][j >> 1], 0, (j & 1) ? 0x4342 : 0x4140); };

  // h1 on columns c = 2..23 (pairs j = 1..11), vertical taps
  uint32_t h1[12];
#pragma unroll
  for (int j = 1; j < 12; ++j) h1[j] = tap6x2b(pr(0, j), pr(1, j), pr(2, j), pr(3, j), pr(4, j), pr(5, j));

  // b1 (row k=2) and s1 (row k=3) at output columns c = 4..19 (pairs j = 2..9), horizontal taps
  uint32_t bc[8], sc[8];
#pragma unroll
  for (int k = 2; k <= 3; ++k) {
    uint32_t p[12];
#pragma unroll
    for (int j = 1; j < 12; ++j) p[j] = pr(k, j);
#pragma unroll
    for (int j = 2; j < 10; ++j) {
      const uint32_t xm1 = __byte_perm(p[j - 1], p[j], 0x5432);     // columns (2j-1, 2j)
      const uint32_t xp1 = __byte_perm(p[j], p[j + 1], 0x5432);     // (2j+1, 2j+2)
      const uint32_t xp3 = __byte_perm(p[j + 1], p[j + 2], 0x5432); // (2j+3, 2j+4)
      const uint32_t v = clip_half2(tap6x2b(p[j - 1], xm1, p[j], xp1, p[j + 1], xp3));
      if (k == 2) bc[j - 2] = v; else sc[j - 2] = v;
    }
  }
  // h and m = h at x+1: clipped h1 on pairs j = 2..10 (columns 4..21)
  uint32_t hc[9];
#pragma unroll
  for (int j = 2; j < 11; ++j) hc[j - 2] = clip_half2(h1[j]);

  // j1 = tap6 over h1 at columns c-2..c+3 (int32), c = 4..19
  int hv[22];
#pragma unroll
  for (int j = 1; j < 12; ++j) { hv[2 * j - 2] = lo_u16(h1[j]); hv[2 * j - 1] = hi_u16(h1[j]); }   // hv[i] = h1 + B at c = i+2
  uint32_t jb[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) {   // output column c = i+4: h1 at c-2..c+3 = hv[i .. i+5]
    const int j1 = (hv[i] + hv[i + 5]) - 5 * (hv[i + 1] + hv[i + 4]) + 20 * (hv[i + 2] + hv[i + 3]);
    jb[i] = clip_j(j1);
  }

  uint32_t Gw[4], Hw[4], Mw[4], bw[4], hw[4], mw[4], sw[4], jw[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    Gw[q] = w[2][q + 1];                                        // columns 4q+4 .. 4q+7
    Hw[q] = __funnelshift_r(w[2][q + 1], w[2][q + 2], 8);       // +1 column
    Mw[q] = w[3][q + 1];                                        // row y+1
    bw[q] = bytes_of(bc[2 * q], bc[2 * q + 1]);
    sw[q] = bytes_of(sc[2 * q], sc[2 * q + 1]);
    hw[q] = bytes_of(hc[2 * q], hc[2 * q + 1]);
    // m: columns 4q+5..4q+8 = hc[2q] hi, hc[2q+1] lo/hi, hc[2q+2] lo
    mw[q] = __byte_perm(bytes_of(hc[2 * q], hc[2 * q + 1]), bytes_of(hc[2 * q + 2], hc[2 * q + 2]), 0x4321);
    jw[q] = __byte_perm(__byte_perm(jb[4 * q], jb[4 * q + 1], 0x0040), __byte_perm(jb[4 * q + 2], jb[4 * q + 3], 0x0040),
                        0x5410);
  }

  const uint32_t kh = P.k_hi;
  uint8_t* dst = P.sf + (size_t)rr * P.pitch + 16 * g;
  auto put = [&](int ph, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    *reinterpret_cast<uint4*>(dst + ph * P.plane) = make_uint4(a, b, c, d);
  };
#define PLANE(ph, EXPR) put(ph, EXPR(0), EXPR(1), EXPR(2), EXPR(3))
#define G_(q) Gw[q]
#define A_(q) vavg4(Gw[q], bw[q], kh)
#define B_(q) bw[q]
#define C_(q) vavg4(Hw[q], bw[q], kh)
#define D_(q) vavg4(Gw[q], hw[q], kh)
#define E_(q) vavg4(bw[q], hw[q], kh)
#define F_(q) vavg4(bw[q], jw[q], kh)
#define Gq_(q) vavg4(bw[q], mw[q], kh)
#define H_(q) hw[q]
#define I_(q) vavg4(hw[q], jw[q], kh)
#define J_(q) jw[q]
#define K_(q) vavg4(jw[q], mw[q], kh)
#define N_(q) vavg4(Mw[q], hw[q], kh)
#define Pq_(q) vavg4(hw[q], sw[q], kh)
#define Q_(q) vavg4(jw[q], sw[q], kh)
#define R_(q) vavg4(mw[q], sw[q], kh)
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

template <bool INTERIOR>
__device__ __forceinline__ void int_body(const IntParams& P, int g, int rr) {
  const int x0 = 16 * g - P.pad, y = rr - P.pad;
  // source rows y-2 .. y+3 (k = 0..5), columns x0-4 .. x0+19 (c = 0..23, 6 words)
  uint32_t w[6][6];
#pragma unroll
  for (int k = 0; k < 6; ++k) {
    const int yy = clampi(y - 2 + k, 0, P.H - 1);
    if (INTERIOR) {
      const uint32_t* src = reinterpret_cast<const uint32_t*>(P.rf + (size_t)yy * P.W + x0 - 4);
#pragma unroll
      for (int q = 0; q < 6; ++q) w[k][q] = __ldg(src + q);
    } else {
#pragma unroll
      for (int q = 0; q < 6; ++q) w[k][q] = load4_clamped(P.rf, P.W, P.H, x0 - 4 + 4 * q, yy);
    }
  }
  int_compute(P, g, rr, w);
}

#ifndef FEVES_INT_MINB
#define FEVES_INT_MINB 1
#endif
__global__ void __launch_bounds__(128, FEVES_INT_MINB) int_subpel_kernel(const IntParams P) {
  if (blockIdx.z == gridDim.z - 1) {
    const int g = P.g_lo + blockIdx.x * blockDim.x + threadIdx.x;
    const int rr = P.row_begin + blockIdx.y * blockDim.y + threadIdx.y;
    if (g < P.g_hi && rr < P.row_end) int_body<true>(P, g, rr);
  } else {
    const int t = threadIdx.y * blockDim.x + threadIdx.x;
    const int bx = P.border_bx, by = (blockDim.x * blockDim.y) / bx;
    const int tb = blockIdx.x * bx + t % bx, tr = t / bx;
    const int groups = P.pitch / 16, nb = groups - (P.g_hi - P.g_lo);
    if (tb >= nb) return;
    const int g = tb < P.g_lo ? tb : P.g_hi + (tb - P.g_lo);
    const int rr = P.row_begin + blockIdx.y * by + tr;
    if (rr < P.row_end) int_body<false>(P, g, rr);
  }
}

// Shared-memory tiled INT: CTA = kIntTx plane groups (16 columns each) x kIntTy plane rows.
// The source tile (kIntTy + 5 rows x 16 kIntTx + 8 columns, clamped, G5) is staged once with
// coalesced 4-byte loads (each source word is read by 6 rows x 1.5 groups in the per-thread
// kernel), then every thread reads its 6 x 6 words with LDS.128 + LDS.64 (its window starts
// 16-byte aligned in the tile, so a warp's quarter-requests are bank-conflict free).
#ifndef FEVES_INT_TX
#define FEVES_INT_TX 8
#endif
#ifndef FEVES_INT_TY
#define FEVES_INT_TY 16
#endif
constexpr int kIntTx = FEVES_INT_TX, kIntTy = FEVES_INT_TY;
constexpr int kIntSrcRows = kIntTy + 5, kIntSrcWords = 4 * kIntTx + 2;
constexpr int kIntStride = (kIntSrcWords + 3) & ~3;                                          // words per tile row
static_assert(kIntStride >= kIntSrcWords && kIntStride % 4 == 0, "INT tile row stride");

#ifndef FEVES_INT_TPC
#define FEVES_INT_TPC 1   // tile rows per CTA (> 1: the next tile is copied while one computes; measured slower: 1 wave)
#endif
__device__ __forceinline__ void int_cp4(uint32_t* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(src));
}

__global__ void __launch_bounds__(kIntTx * kIntTy) int_tile_kernel(const IntParams P) {
  __shared__ __align__(16) uint32_t tile[2][kIntSrcRows * kIntStride];
  const int groups = P.pitch / 16;
  const int g0 = kIntTx * blockIdx.x;
  const int xs = 16 * g0 - P.pad - 4;                      // frame column of tile word 0
  const int tid = threadIdx.y * kIntTx + threadIdx.x;
  const bool fast = P.vec_ok && xs >= 0 && xs + 4 * kIntSrcWords <= P.W;
  // stage the source tile of tile row ty (plane rows r0 .. r0+15) into buffer b.  Border tiles
  // with aligned rows (vec_ok: W % 4 == 0, so a word is wholly inside or wholly outside the
  // frame) copy the frame's edge word in place of every outside word, and edge_fix() then
  // replicates its edge byte (G5 clamp) -- all loads stay asynchronous; the per-word clamped
  // loads (a dependent global round trip per item) are left to unaligned frames only.
  auto stage = [&](int ty, int b) {
    const int ys = P.row_begin + kIntTy * ty - P.pad - 2;
    for (int i = tid; i < kIntSrcRows * kIntSrcWords; i += kIntTx * kIntTy) {
      const int r = i / kIntSrcWords, q = i - r * kIntSrcWords;
      const int yy = clampi(ys + r, 0, P.H - 1);
      uint32_t* d = &tile[b][r * kIntStride + q];
      if (fast) {
        int_cp4(d, reinterpret_cast<const uint32_t*>(P.rf + (size_t)yy * P.W + xs) + q);
      } else if (P.vec_ok) {
        const int x = min(max(xs + 4 * q, 0), P.W - 4);      // the edge word for outside words
        int_cp4(d, P.rf + (size_t)yy * P.W + x);
      } else {
        *d = load4_clamped(P.rf, P.W, P.H, xs + 4 * q, yy);
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  // after this thread's copies of buffer b landed: outside words = their edge byte x 4
  auto edge_fix = [&](int b) {
    if (fast || !P.vec_ok) return;
    for (int i = tid; i < kIntSrcRows * kIntSrcWords; i += kIntTx * kIntTy) {
      const int r = i / kIntSrcWords, q = i - r * kIntSrcWords;
      const int x = xs + 4 * q;
      uint32_t* d = &tile[b][r * kIntStride + q];
      if (x < 0) *d = 0x01010101u * (*d & 0xffu);                 // column 0
      else if (x + 4 > P.W) *d = 0x01010101u * (*d >> 24);        // column W - 1
    }
  };
  const int n_ty = (P.row_end - P.row_begin + kIntTy - 1) / kIntTy;
  const int ty0 = FEVES_INT_TPC * blockIdx.y, ty1 = min(n_ty, ty0 + FEVES_INT_TPC);
  stage(ty0, 0);
  for (int ty = ty0; ty < ty1; ++ty) {
    const int b = (ty - ty0) & 1;
    if (ty + 1 < ty1) {
      stage(ty + 1, b ^ 1);                                  // in flight during this tile's compute
      asm volatile("cp.async.wait_group 1;" ::: "memory");
    } else {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    edge_fix(b);
    __syncthreads();
    const int g = g0 + threadIdx.x, rr = P.row_begin + kIntTy * ty + threadIdx.y;
    if (g < groups && rr < P.row_end) {
      uint32_t w[6][6];
#pragma unroll
      for (int k = 0; k < 6; ++k) {
        const uint32_t* t = tile[b] + (threadIdx.y + k) * kIntStride + 4 * threadIdx.x;
        const uint4 a4 = *reinterpret_cast<const uint4*>(t);
        const uint2 b2 = *reinterpret_cast<const uint2*>(t + 4);
        w[k][0] = a4.x; w[k][1] = a4.y; w[k][2] = a4.z; w[k][3] = a4.w; w[k][4] = b2.x; w[k][5] = b2.y;
      }
      int_compute(P, g, rr, w);
    }
    __syncthreads();                                         // buffer b is restaged two tiles later
  }
}

}  // namespace feves
