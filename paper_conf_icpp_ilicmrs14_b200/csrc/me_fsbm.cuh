// me_fsbm.cuh -- integer full-search block-matching ME for sm_100a.
//
// P:6: "the best matching candidate for the currently processed MB is found
// within the predefined search areas (SAs) in previously encoded RFs ... 7
// partitioning modes ... minimum distortion value ... SAD".
//
// One CTA = one 16x16 MB, looping over its n_rf reference frames.  Per RF:
//  a1  the SA window ((S+15) x (S+15) bytes around the MB, clamped at the frame
//      edge, G5) is staged in shared memory as FOUR byte-shifted copies so that
//      every candidate row is read with 4-byte aligned LDS.32;
//  a2  lane = one horizontal displacement dx (32 consecutive dx per warp, so the
//      4 copies x 8 words of a warp's reads hit 32 distinct banks); the lane
//      sweeps dy vertically, T = 4 candidates at a time, so each staged RF row
//      is loaded once and reused by 4 candidates (19 rows for 4 candidates).
//      The 16 CF rows of the MB live in 64 registers.  Each 4x4 SAD is 4
//      chained VABSDIFF4.ACC (one instruction per 4 px, ALU pipe);
//  a3  aggregation is done directly in KEY space on the FMA pipe:
//      key(child) = sad<<16 | rank, key(parent) = IMAD(sad(other child), 2^16,
//      key(child)) -- one IMAD per partition, no ALU op;
//  a4  per partition a running minimum of keys; two candidates per 3-input
//      VIMNMX3 (ALU).  key = SAD * 2^16 + spiral rank (G4) makes the argmin
//      unique and independent of the reduction order.  Warp: CREDUX.MIN
//      (__reduce_min_sync); CTA: shared memory; rank -> (dx,dy) by table.
// Roofline: ALU pipe = 64 lanes/clk/SM for VABSDIFF4, VIMNMX3,
// IADD3 (measured, profiles/r01/int_peaks.json); per MB-candidate 64
// VABSDIFF4 + 20.5 VIMNMX3 on ALU, ~55 IMAD on FMA.
#pragma once
#include "common.cuh"

namespace feves {

constexpr int kMeT = 4;   // candidates per vertical step

struct MeParams {
  const uint8_t* cf;
  const uint8_t* rf[kMaxRf];
  int W, H, S, R, n_rf;       // n_rf = RFs searched by this launch (RF ramp)
  int rf_stride;              // RF dimension of the output layout (the context's n_rf)
  int mb_cols, row0;
  const uint32_t* rank_tab;   // [S][S], [dy+R][dx+R] -> spiral rank (G4)
  const uint32_t* inv_tab;    // rank -> (dx & 0xffff) | (dy << 16)
  int16_t* out_mvs;
  uint16_t* out_sads;
  int lx, ngx, nsub, nwy, dyl;  // lane / warp geometry (see me_geometry())
  int pw, cstride;              // shared window: words per row, words per copy
};

// Per-candidate aggregation state carried between 4x4 block rows.
struct RowState {
  uint32_t k4prev[4];   // keys of the previous block row's 4x4s
  uint32_t p84top[2];   // SADs of the upper 8x4 pair (for 8x8)
  uint32_t k84top[2];   // keys of the upper 8x4 pair (for 8x8)
  uint32_t p88top[2];   // SADs of the top 8x8 pair (for 8x16)
  uint32_t p168top;     // SAD of the top 16x8 (for 16x16)
};

constexpr uint32_t kSh = 65536u;

// Keys of every partition completed by 4x4 block row BY of one candidate.
// L = the four 4x4 SADs of this block row.  Slot -> partition map: part_of().
template <int BY>
__device__ __forceinline__ void block_row_keys(const uint32_t (&L)[4], uint32_t rank, RowState& st,
                                               uint32_t (&K)[16]) {
  uint32_t k4[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) k4[i] = L[i] * kSh + rank;
  const uint32_t p84_0 = L[0] + L[1], p84_1 = L[2] + L[3];
  const uint32_t k84_0 = L[1] * kSh + k4[0], k84_1 = L[3] * kSh + k4[2];
#pragma unroll
  for (int i = 0; i < 4; ++i) K[i] = k4[i];
  K[4] = k84_0;
  K[5] = k84_1;
  if ((BY & 1) == 0) {
#pragma unroll
    for (int i = 0; i < 4; ++i) st.k4prev[i] = k4[i];
    st.p84top[0] = p84_0; st.p84top[1] = p84_1;
    st.k84top[0] = k84_0; st.k84top[1] = k84_1;
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i) K[6 + i] = L[i] * kSh + st.k4prev[i];      // 4x8
    const uint32_t k88_0 = p84_0 * kSh + st.k84top[0];                      // 8x8
    const uint32_t k88_1 = p84_1 * kSh + st.k84top[1];
    K[10] = k88_0;
    K[11] = k88_1;
    const uint32_t p88_0 = p84_0 + st.p84top[0], p88_1 = p84_1 + st.p84top[1];
    const uint32_t k168 = p88_1 * kSh + k88_0;                             // 16x8
    K[12] = k168;
    if (BY == 1) {
      st.p88top[0] = p88_0; st.p88top[1] = p88_1;
      st.p168top = p88_0 + p88_1;
    } else {
      K[13] = st.p88top[0] * kSh + k88_0;                                   // 8x16 left
      K[14] = st.p88top[1] * kSh + k88_1;                                   // 8x16 right
      K[15] = st.p168top * kSh + k168;                                      // 16x16
    }
  }
}

// partition index (G7) of slot `slot` of block row `by`; -1 = unused
__host__ __device__ constexpr int part_of(int by, int slot) {
  // sub-MBs of this block row: s0 = (by/2)*2 (left), s0+1 (right); k-row = by&1
  return slot < 4 ? 25 + 4 * ((by / 2) * 2 + slot / 2) + (by & 1) * 2 + (slot & 1)     // 4x4
       : slot < 6 ? 9 + 2 * ((by / 2) * 2 + (slot - 4)) + (by & 1)                      // 8x4
       : (by & 1) == 0 ? -1
       : slot < 10 ? 17 + 2 * ((by / 2) * 2 + (slot - 6) / 2) + ((slot - 6) & 1)        // 4x8
       : slot < 12 ? 5 + (by / 2) * 2 + (slot - 10)                                      // 8x8
       : slot == 12 ? 1 + by / 2                                                         // 16x8
       : by != 3 ? -1
       : slot == 13 ? 3 : slot == 14 ? 4 : 0;                                            // 8x16, 16x16
}

__device__ __forceinline__ uint32_t umin3(uint32_t a, uint32_t b, uint32_t c) { return min(min(a, b), c); }

template <int BY>
__device__ __forceinline__ void fold_pair(uint32_t (&M)[kNPart], const uint32_t (&Ka)[16], const uint32_t (&Kb)[16]) {
#pragma unroll
  for (int s = 0; s < 16; ++s) {
    const int p = part_of(BY, s);
    if (p >= 0) M[p] = umin3(M[p], Ka[s], Kb[s]);
  }
}

__global__ void __launch_bounds__(256) me_fsbm_kernel(const MeParams P) {
  extern __shared__ uint32_t smem[];
  uint32_t* win = smem;                                   // 4 copies x cstride words
  uint32_t* red = smem + 4 * P.cstride;                   // [nwarps][41]

  const int mbx = blockIdx.x, mby = P.row0 + blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  const int R = P.R, S = P.S;

  // ---- lane geometry: dx column and dy sub-range ----
  const int gx = warp % P.ngx, wyi = warp / P.ngx;
  const int xi = lane % P.lx, sub = lane / P.lx;
  const int dx = min(-R + gx * P.lx + xi, R - 1);          // beyond-range lanes duplicate dx=R-1
  const int off = dx + R;                                  // byte offset inside the window row
  const uint32_t* wbase = win + (off & 3) * P.cstride + (off >> 2);
  const int dy_begin = -R + (wyi * P.nsub + sub) * P.dyl;

  // ---- CF MB in registers: cf[row][4 words] ----
  uint32_t cfw[16][4];
#pragma unroll
  for (int r = 0; r < 16; ++r)
#pragma unroll
    for (int b = 0; b < 4; ++b) cfw[r][b] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * b, 16 * mby + r);

  const int xw0 = 16 * mbx - R, yw0 = 16 * mby - R;
  const int win_rows = S + 15;

  for (int ref = 0; ref < P.n_rf; ++ref) {
    const uint8_t* __restrict__ rf = P.rf[ref];
    __syncthreads();
    // ---- a1: stage 4 byte-shifted copies of the SA window ----
    for (int item = threadIdx.x; item < win_rows * P.pw; item += blockDim.x) {
      const int row = item / P.pw, q = item - row * P.pw;
      const uint32_t lo = load4_clamped(rf, P.W, P.H, xw0 + 4 * q, yw0 + row);
      const uint32_t hi = load4_clamped(rf, P.W, P.H, xw0 + 4 * q + 4, yw0 + row);
      uint32_t* dst = win + row * P.pw + q;
      dst[0] = lo;
      dst[P.cstride] = __byte_perm(lo, hi, 0x4321);
      dst[2 * P.cstride] = __byte_perm(lo, hi, 0x5432);
      dst[3 * P.cstride] = __byte_perm(lo, hi, 0x6543);
    }
    __syncthreads();

    uint32_t M[kNPart];
#pragma unroll
    for (int p = 0; p < kNPart; ++p) M[p] = 0xffffffffu;

    const uint32_t* rank_col = P.rank_tab + off;
    for (int c = 0; c < P.dyl; c += kMeT) {
      const int dy0 = min(dy_begin + c, R - kMeT);        // clamped chunk: duplicates are harmless
      uint32_t rank[kMeT];
#pragma unroll
      for (int t = 0; t < kMeT; ++t) rank[t] = __ldg(rank_col + (dy0 + t + R) * S);
      const uint32_t* wrow = wbase + (dy0 + R) * P.pw;

      uint32_t acc[kMeT][4];
      RowState st[kMeT];
      uint32_t Kp[kMeT][16];
#pragma unroll
      for (int i = 0; i < kMeT + 15; ++i) {
        uint32_t w[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) w[b] = wrow[i * P.pw + b];
#pragma unroll
        for (int t = 0; t < kMeT; ++t) {
          const int r = i - t;                              // CF row paired with RF row i
          if (r >= 0 && r < 16) {
#pragma unroll
            for (int b = 0; b < 4; ++b) acc[t][b] = vad4(cfw[r][b], w[b], (r & 3) ? acc[t][b] : 0u);
            if ((r & 3) == 3) {
              const int by = r >> 2;
              if (by == 0) block_row_keys<0>(acc[t], rank[t], st[t], Kp[t]);
              if (by == 1) block_row_keys<1>(acc[t], rank[t], st[t], Kp[t]);
              if (by == 2) block_row_keys<2>(acc[t], rank[t], st[t], Kp[t]);
              if (by == 3) block_row_keys<3>(acc[t], rank[t], st[t], Kp[t]);
              if (t & 1) {                                  // pair (t-1, t) finished this block row
                if (by == 0) fold_pair<0>(M, Kp[t - 1], Kp[t]);
                if (by == 1) fold_pair<1>(M, Kp[t - 1], Kp[t]);
                if (by == 2) fold_pair<2>(M, Kp[t - 1], Kp[t]);
                if (by == 3) fold_pair<3>(M, Kp[t - 1], Kp[t]);
              }
            }
          }
        }
      }
    }

    // ---- a4: warp min (CREDUX), then CTA min through shared memory ----
#pragma unroll
    for (int p = 0; p < kNPart; ++p) {
      const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
      if (lane == 0) red[warp * kNPart + p] = v;
    }
    __syncthreads();
    for (int p = threadIdx.x; p < kNPart; p += blockDim.x) {
      uint32_t k = red[p];
      for (int w = 1; w < nwarps; ++w) k = min(k, red[w * kNPart + p]);
      const uint32_t mv = __ldg(P.inv_tab + (k & 0xffffu));
      const size_t o = ((size_t)(blockIdx.y * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
      reinterpret_cast<uint32_t*>(P.out_mvs)[o] = mv;
      P.out_sads[o] = (uint16_t)(k >> 16);
    }
  }
}

}  // namespace feves
