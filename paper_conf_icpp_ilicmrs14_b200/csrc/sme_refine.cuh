// sme_refine.cuh -- SME: sub-pixel refinement of the ME MVs.
//
// P:6: "By relying on the MVs from the ME and the SFs from the INT, the
// Sub-Pixel Motion Estimation (SME) is applied to further refine the MVs";
// "the MVs from ME define the initial search point for the SME".
// Algorithm (O3, G12-G14): centre c = 4*mv (cost = ME SAD); half
// stage: the 8 ring-1 neighbours c + 2*s_k in spiral order, update on strict
// <; quarter stage: the 8 neighbours of the best half position, strict <.
//
// 16 lanes = the 16 4x4 blocks of one (MB, RF).  Lane bits (bx0, by0, bx1,
// by1) make every partition of every mode an xor-closed lane set, so each
// partition's SAD is a butterfly all-reduce over that mode's bits and every
// lane of a partition holds the same (best, bestv) -- no divergence.  Each
// lane computes, per mode and candidate, the SAD of its own 4x4 block against
// the SF phase plane (4 rows x one unaligned 4-byte window, VABSDIFF4.ACC).
#pragma once
#include "common.cuh"

namespace feves {

struct SmeParams {
  const uint8_t* cf;
  const uint8_t* sf[kMaxRf];
  const uint32_t* in_mvs;     // int16 pairs as u32
  const uint16_t* in_sads;    // may be null
  uint32_t* out_qmvs;
  uint16_t* out_sads;
  int W, H, n_rf, rf_stride, mb_cols, row0, n_items;   // n_rf RFs refined, rf_stride = layout
  int pad, pitch;
  size_t plane;
};

__constant__ int8_t c_ring1[8][2] = {{0, -1}, {0, 1}, {-1, -1}, {1, -1}, {-1, 0}, {1, 0}, {-1, 1}, {1, 1}};

// 4x4 SAD of this lane's CF block against SF samples at quarter-pel offset v
__device__ __forceinline__ uint32_t block_sad_q(const uint8_t* __restrict__ sf, size_t plane, int pitch,
                                                int pad, int bxp, int byp, int vx, int vy,
                                                const uint32_t (&cfb)[4]) {
  const uint8_t* pl = sf + (size_t)(4 * (vy & 3) + (vx & 3)) * plane;
  const int X = bxp + (vx >> 2) + pad, Y = byp + (vy >> 2) + pad;
  const uint8_t* p0 = pl + (size_t)Y * pitch + X;
  const uintptr_t a = reinterpret_cast<uintptr_t>(p0);
  const uint32_t* w = reinterpret_cast<const uint32_t*>(a & ~uintptr_t(3));
  const uint32_t sh = 8u * (uint32_t)(a & 3);
  const int wp = pitch >> 2;
  uint32_t s = 0;
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const uint32_t lo = __ldg(w + r * wp), hi = __ldg(w + r * wp + 1);
    s = vad4(cfb[r], __funnelshift_r(lo, hi, sh), s);
  }
  return s;
}

// all-reduce over the xor-closed lane set of one partition (offsets < 16 stay
// inside the 16-lane half that owns this (MB, RF))
template <int MASK>
__device__ __forceinline__ uint32_t part_sum(uint32_t v) {
  const unsigned half = (threadIdx.x & 16) ? 0xffff0000u : 0x0000ffffu;
  if (MASK & 1) v += __shfl_xor_sync(half, v, 1);
  if (MASK & 2) v += __shfl_xor_sync(half, v, 2);
  if (MASK & 4) v += __shfl_xor_sync(half, v, 4);
  if (MASK & 8) v += __shfl_xor_sync(half, v, 8);
  return v;
}

template <int MASK>
__device__ __forceinline__ void refine_mode(const SmeParams& P, const uint8_t* __restrict__ sf, int p, size_t o,
                                            int bxp, int byp, int b, const uint32_t (&cfb)[4]) {
  const uint32_t mv = __ldg(P.in_mvs + o + p);
  const int cx = 4 * (int)(int16_t)(mv & 0xffffu), cy = 4 * (int)(int16_t)(mv >> 16);
  uint32_t best = P.in_sads ? (uint32_t)__ldg(P.in_sads + o + p)
                            : part_sum<MASK>(block_sad_q(sf, P.plane, P.pitch, P.pad, bxp, byp, cx, cy, cfb));
  int bvx = cx, bvy = cy;
#pragma unroll
  for (int k = 0; k < 8; ++k) {              // half-pel ring around c
    const int vx = cx + 2 * c_ring1[k][0], vy = cy + 2 * c_ring1[k][1];
    const uint32_t s = part_sum<MASK>(block_sad_q(sf, P.plane, P.pitch, P.pad, bxp, byp, vx, vy, cfb));
    if (s < best) { best = s; bvx = vx; bvy = vy; }
  }
  const int hx = bvx, hy = bvy;
#pragma unroll
  for (int k = 0; k < 8; ++k) {              // quarter-pel ring around the best half position
    const int vx = hx + c_ring1[k][0], vy = hy + c_ring1[k][1];
    const uint32_t s = part_sum<MASK>(block_sad_q(sf, P.plane, P.pitch, P.pad, bxp, byp, vx, vy, cfb));
    if (s < best) { best = s; bvx = vx; bvy = vy; }
  }
  if ((b & MASK) == 0) {                     // partition leader writes
    P.out_qmvs[o + p] = (uint32_t)(uint16_t)bvx | ((uint32_t)(uint16_t)bvy << 16);
    P.out_sads[o + p] = (uint16_t)best;
  }
}

__global__ void __launch_bounds__(128) sme_refine_kernel(const SmeParams P) {
  const int item = blockIdx.x * (blockDim.x >> 4) + (threadIdx.x >> 4);
  if (item >= P.n_items) return;             // whole 16-lane groups exit together
  const int b = threadIdx.x & 15;
  const int bx0 = b & 1, by0 = (b >> 1) & 1, bx1 = (b >> 2) & 1, by1 = (b >> 3) & 1;
  const int bx = 2 * bx1 + bx0, by = 2 * by1 + by0;
  const int ref = item % P.n_rf, mbi = item / P.n_rf;
  const int mbx = mbi % P.mb_cols, mby = P.row0 + mbi / P.mb_cols;
  const int bxp = 16 * mbx + 4 * bx, byp = 16 * mby + 4 * by;
  uint32_t cfb[4];
#pragma unroll
  for (int r = 0; r < 4; ++r) cfb[r] = load4_clamped(P.cf, P.W, P.H, bxp, byp + r);
  const uint8_t* __restrict__ sf = P.sf[ref];
  const size_t o = ((size_t)mbi * P.rf_stride + ref) * kNPart;    // [mb][ref][41]
  const int s = 2 * by1 + bx1;
  refine_mode<15>(P, sf, 0, o, bxp, byp, b, cfb);                           // 16x16
  refine_mode<7>(P, sf, 1 + by1, o, bxp, byp, b, cfb);                      // 16x8
  refine_mode<11>(P, sf, 3 + bx1, o, bxp, byp, b, cfb);                     // 8x16
  refine_mode<3>(P, sf, 5 + s, o, bxp, byp, b, cfb);                        // 8x8
  refine_mode<1>(P, sf, 9 + 2 * s + by0, o, bxp, byp, b, cfb);              // 8x4
  refine_mode<2>(P, sf, 17 + 2 * s + bx0, o, bxp, byp, b, cfb);             // 4x8
  refine_mode<0>(P, sf, 25 + 4 * s + 2 * by0 + bx0, o, bxp, byp, b, cfb);   // 4x4
}

}  // namespace feves
