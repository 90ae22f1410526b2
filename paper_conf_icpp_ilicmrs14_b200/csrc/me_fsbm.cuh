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
//  a3  aggregation is done directly in KEY space on the FMA pipe: key(4x4) =
//      sad<<16 | rank; S <= 64 (and S = 128 quadrant by quadrant): key(parent) =
//      key(child a) + key(child b) with the dense rank (SumKeys, below); otherwise
//      key(parent) = IMAD(sad(other child), 2^KSH, key(child)).  One IMAD per
//      partition, no ALU op;
//  a4  per partition a running minimum of keys; two candidates per 3-input
//      VIMNMX3 (ALU).  key = SAD * 2^16 + spiral rank (G4) makes the argmin
//      unique and independent of the reduction order.  Warp: CREDUX.MIN
//      (__reduce_min_sync); CTA: shared memory; rank -> (dx,dy) by table.
// Roofline: ALU pipe = 64 lanes/clk/SM for VABSDIFF4, VIMNMX3,
// IADD3 (measured, profiles/r01/int_peaks.json); per MB-candidate 64
// VABSDIFF4 + 20.5 VIMNMX3 on ALU, 41 IMAD on FMA (key-sum; 54 otherwise).
#pragma once
#include "common.cuh"

namespace feves {

#ifndef FEVES_ME_T
#define FEVES_ME_T 4
#endif
#ifndef FEVES_ME_MINB
#define FEVES_ME_MINB 4
#endif
constexpr int kMeT = FEVES_ME_T;   // candidates per vertical step

struct MeParams {
  const uint8_t* cf;
  const uint8_t* rf[kMaxRf];
  int W, H, S, R, n_rf;       // S = candidates per axis (sa_range, +1 if inclusive); n_rf = RFs searched
  int rf_stride;              // RF dimension of the output layout (the context's n_rf)
  int mb_cols, row0;
  const uint32_t* rank_tab;   // [S][Sp] (S candidates per axis), [dx+R][dy+R] -> key addend E =
                              // lambda*R(4dx,4dy)*kmul + spiral rank (G4, G18)
  const uint32_t* inv_tab;    // rank -> (dx & 0xffff) | (dy << 16)
  const uint32_t* glob_tab;   // S = 128 quadrant key-sum: [quadrant][local rank] -> global dense rank
  uint32_t kmul;              // key = J * kmul + rank: 2^16 (lambda = 0) or 2^15 (J may exceed 16 bits)
  int kshift, lambda;
  int16_t* out_mvs;
  uint16_t* out_sads;
  const int16_t* pmv;         // G21 predictor [frame MB][rf_stride][2] integer-pel (runtime-S kernel only), or null
  int max_pmv;                // G21 clamp of each predictor component
  int vec_ok;                 // 16-byte aligned rows and window start: vector staging allowed
  int rf_per_cta;             // RFs searched per CTA: CTA (x, y, z) takes RFs [z * rf_per_cta, +rf_per_cta)
  // fused SME (template FUSE): SF of each RF, quarter-pel outputs
  const uint8_t* sf[kMaxRf];
  int sf_pad, sf_pitch;
  size_t sf_plane;
  uint32_t* out_qmvs;
  uint16_t* out_qsads;
};

// ---- launch geometry, shared by host and device (compile-time for the template sizes) ----
__host__ __device__ constexpr int me_lx(int S) { return S >= 32 ? 32 : S >= 16 ? 16 : S >= 8 ? 8 : 4; }
__host__ __device__ constexpr int me_ngx(int S) { return (S + me_lx(S) - 1) / me_lx(S); }
__host__ __device__ constexpr int me_nsub(int S) { return 32 / me_lx(S); }
// warps splitting the dy range: at S = 16 (CIF, 396 MBs, one RF) a second warp takes the
// other half of the dy range, doubling the warps of a grid too small to fill the GPU
// (ME 10.9 -> 9.0 us).  Measured slower for S = 32 (69.9 -> 73.4 us), so only S = 16.
#ifndef FEVES_ME_NWY64
#define FEVES_ME_NWY64 1
#endif
#ifndef FEVES_ME_NWY32
#define FEVES_ME_NWY32 1
#endif
__host__ __device__ constexpr int me_nwy(int S) { return S == 16 ? 2 : S == 32 ? FEVES_ME_NWY32 : S == 64 ? FEVES_ME_NWY64 : 1; }
__host__ __device__ constexpr int me_dyl(int S) {
  return ((S + me_nsub(S) * me_nwy(S) - 1) / (me_nsub(S) * me_nwy(S)) + kMeT - 1) / kMeT * kMeT;
}
__host__ __device__ constexpr int me_pw(int S) { return (((S - 1) >> 2) + 4 + 3) & ~3; }   // words/row, %4 == 0
// window rows staged at once: the whole (S+15)-row window, or at S = 128 one dy half of it
// (S/2 + 15 rows; the window then costs 46 KB instead of 82 KB of shared memory per CTA,
// so 4 CTAs = 16 warps fit per SM instead of 2 CTAs = 8 warps)
__host__ __device__ constexpr int me_nstage(int S) { return S == 128 ? 2 : 1; }
__host__ __device__ constexpr int me_win_rows(int S) { return S / me_nstage(S) + 15; }
__host__ __device__ constexpr int me_cstride(int S) {                                      // == 8 (mod 32)
  return me_win_rows(S) * me_pw(S) + ((8 - (me_win_rows(S) * me_pw(S)) % 32) % 32 + 32) % 32;
}
// rank table column pitch: a lane's T = 4 consecutive dy are one aligned 16-byte load
__host__ __device__ constexpr int me_rank_pitch(int S) { return (S + 3) & ~3; }
__host__ __device__ constexpr int me_threads(int S) { return 32 * me_ngx(S) * me_nwy(S); }
// reduction buffer: [nwarps][halves][41]; two dy halves at S = 128 (QuadKeys)
__host__ __device__ constexpr int me_red_halves(int S) { return S == 128 ? 2 : 1; }
__host__ __device__ constexpr int me_smem_words(int S) {
  return 64 + 4 * me_cstride(S) + (me_threads(S) / 32) * me_red_halves(S) * kNPart;
}
// + fused SME: the ME winners of every RF (packed MV, SAD) stay in shared memory
__host__ __device__ constexpr int me_smem_words_fused(int S, int n_rf) { return me_smem_words(S) + 2 * n_rf * kNPart; }

// Per-candidate aggregation state carried between 4x4 block rows.
struct RowState {
  uint32_t k4prev[4];   // keys of the previous block row's 4x4s (for 4x8)
  uint32_t p84top[2];   // SADs of the upper 8x4 pair (for 8x8)
  uint32_t p88top[2];   // SADs of the top 8x8 pair (for 8x16)
  uint32_t p168top;     // SAD of the top 16x8 (for 16x16)
};

constexpr uint32_t kSh = 65536u;

// Keys of every partition completed by 4x4 block row BY of one candidate.
// L = the four 4x4 SADs of this block row; key = SAD * 2^16 + rank.  Every key
// is ONE IMAD (FMA pipe) on a child's SAD or key; plain sums are IMAD.IADD.
// key(parent) = sad(other child) * 2^KSH + key(child): one IMAD with an immediate.
// Written as inline PTX so the compiler cannot re-associate it into add-then-IMAD.
template <int KSH>
__device__ __forceinline__ uint32_t kmad(uint32_t sad, uint32_t key) {
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(sad), "n"(1 << KSH), "r"(key));
  return d;
}

// G18: Exp-Golomb se(v) bit length, R(mv) = se(mv.x) + se(mv.y) (quarter-pel)
__host__ __device__ __forceinline__ int se_bits(int v) {
  const unsigned k = v > 0 ? 2u * (unsigned)v - 1u : 2u * (unsigned)(-v);
#ifdef __CUDA_ARCH__
  return 2 * (31 - __clz((int)(k + 1u))) + 1;
#else
  int n = 0;
  while ((k + 1u) >> (n + 1)) ++n;
  return 2 * n + 1;
#endif
}

// plain SAD sum kept on the FMA pipe: the ALU pipe is the bottleneck, and an
// IMAD by an opaque 1 (g_one, a kernel-lifetime register) cannot be fused by
// ptxas into a 3-input IADD3 on the ALU pipe.
__device__ __forceinline__ uint32_t fadd(uint32_t a, uint32_t b, uint32_t one) {
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
  return d;
}

template <int BY, int KSH>
__device__ __forceinline__ void block_row_keys(const uint32_t (&L)[4], uint32_t rank, RowState& st,
                                               uint32_t (&K)[16], uint32_t one) {
  uint32_t k4[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) k4[i] = kmad<KSH>(L[i], rank);                   // 4x4
#pragma unroll
  for (int i = 0; i < 4; ++i) K[i] = k4[i];
  K[4] = kmad<KSH>(L[1], k4[0]);                                                // 8x4
  K[5] = kmad<KSH>(L[3], k4[2]);
  const uint32_t p84_0 = fadd(L[0], L[1], one), p84_1 = fadd(L[2], L[3], one);
  if ((BY & 1) == 0) {
#pragma unroll
    for (int i = 0; i < 4; ++i) st.k4prev[i] = k4[i];
    st.p84top[0] = p84_0; st.p84top[1] = p84_1;
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i) K[6 + i] = kmad<KSH>(L[i], st.k4prev[i]);      // 4x8
    const uint32_t p88_0 = fadd(p84_0, st.p84top[0], one), p88_1 = fadd(p84_1, st.p84top[1], one);
    const uint32_t k88_0 = kmad<KSH>(p88_0, rank), k88_1 = kmad<KSH>(p88_1, rank);  // 8x8
    K[10] = k88_0;
    K[11] = k88_1;
    const uint32_t k168 = kmad<KSH>(p88_1, k88_0);                              // 16x8
    K[12] = k168;
    if (BY == 1) {
      st.p88top[0] = p88_0; st.p88top[1] = p88_1;
      st.p168top = fadd(p88_0, p88_1, one);
    } else {
      K[13] = kmad<KSH>(st.p88top[0], k88_0);                                    // 8x16 left
      K[14] = kmad<KSH>(st.p88top[1], k88_1);                                    // 8x16 right
      K[15] = kmad<KSH>(st.p168top, k168);                                       // 16x16
    }
  }
}

// Key-sum aggregation (S <= 64, pure SAD): with the DENSE spiral rank r < 4096
// (feves_me.cu) the key of a partition made of n 4x4 blocks is the SUM of its
// children's keys, (sum SAD) * 2^16 + n*r with n*r <= 16 * 4095 < 2^16: no carry
// into the SAD field, and for a fixed partition (fixed n) the order of the keys is
// still (SAD, rank).  Every parent key is then ONE IMAD (key_a * 1 + key_b, FMA
// pipe, opaque 1) and no plain SAD sum is needed: 41 FMA-pipe ops per candidate
// instead of 54.  The rank is recovered as (key & 0xffff) >> log2(n).
// S = 128 (16384 candidates) runs the same scheme QUADRANT by quadrant: the rank table
// then holds each candidate's dense rank INSIDE its quadrant (dx < 0 / >= 0, dy < 0 / >= 0;
// 4096 each, in spiral order), a warp's dx all lie in one quadrant column, and the dy sweep
// is cut at dy = 0; after each half the warp minima are stored and the CTA epilogue maps
// (quadrant, local rank) -> global dense rank (glob_tab) and compares SAD * 2^14 + global
// rank (SAD < 2^16, rank < 2^14: 30 bits) -- the same (SAD, spiral rank) order (G4).
template <int S_CT, int KSH>
struct SumKeys { static constexpr bool value = S_CT > 0 && S_CT <= 128 && KSH == 16; };
template <int S_CT, int KSH>
struct QuadKeys { static constexpr bool value = SumKeys<S_CT, KSH>::value && S_CT == 128; };

__host__ __device__ constexpr int part_log2n(int p) {   // log2(number of 4x4 blocks of partition p, G7)
  return p == 0 ? 4 : p < 5 ? 3 : p < 9 ? 2 : p < 25 ? 1 : 0;
}

template <int BY>
__device__ __forceinline__ void block_row_keys_sum(const uint32_t (&L)[4], uint32_t rank, RowState& st,
                                                   uint32_t (&K)[16], uint32_t one) {
  uint32_t k4[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) k4[i] = kmad<16>(L[i], rank);                     // 4x4: n = 1
#pragma unroll
  for (int i = 0; i < 4; ++i) K[i] = k4[i];
  K[4] = fadd(k4[0], k4[1], one);                                               // 8x4: n = 2
  K[5] = fadd(k4[2], k4[3], one);
  if ((BY & 1) == 0) {
#pragma unroll
    for (int i = 0; i < 4; ++i) st.k4prev[i] = k4[i];
    st.p84top[0] = K[4]; st.p84top[1] = K[5];                                   // (keys here)
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i) K[6 + i] = fadd(k4[i], st.k4prev[i], one);     // 4x8: n = 2
    const uint32_t k88_0 = fadd(K[4], st.p84top[0], one), k88_1 = fadd(K[5], st.p84top[1], one);  // 8x8: 4
    K[10] = k88_0;
    K[11] = k88_1;
    const uint32_t k168 = fadd(k88_0, k88_1, one);                              // 16x8: n = 8
    K[12] = k168;
    if (BY == 1) {
      st.p88top[0] = k88_0; st.p88top[1] = k88_1;
      st.p168top = k168;
    } else {
      K[13] = fadd(st.p88top[0], k88_0, one);                                   // 8x16: n = 8
      K[14] = fadd(st.p88top[1], k88_1, one);
      K[15] = fadd(st.p168top, k168, one);                                      // 16x16: n = 16
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

// fold the keys of a candidate pair into the running minima: one VIMNMX3 per partition
template <int BY>
__device__ __forceinline__ void fold_pair(uint32_t (&M)[kNPart], const uint32_t (&Ka)[16], const uint32_t (&Kb)[16]) {
#pragma unroll
  for (int s = 0; s < 16; ++s) {
    const int p = part_of(BY, s);
    if (p >= 0) M[p] = umin3(M[p], Ka[s], Kb[s]);
  }
}

// shared-memory loads the compiler may not hoist out of the candidate loop
// (keeps CF rows out of uniform registers / long-lived registers)
__device__ __forceinline__ uint4 lds128_v(const uint32_t* p) {
  uint4 v;
  const unsigned a = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}


// ---------------------------------------------------------------- fused SME --
// After the ME of its MB, the CTA refines the 41 x n_rf MVs itself (O3; P:86
// "the MVs from ME define the initial search point for the SME"): 16 lanes per
// RF, lane = one 4x4 block (bits bx0, by0, bx1, by1 so every partition of every
// mode is an xor-closed lane set), CF from shared memory, SF from L2/HBM.  The
// SME phase is memory-latency-bound and the ME phase ALU-bound, so while one CTA
// refines, the other resident CTAs of the SM keep the ALU pipe busy.
// ring-1 spiral order s_k (G12/G14): (0,-1),(0,1),(-1,-1),(1,-1),(-1,0),(1,0),(-1,1),(1,1)
__host__ __device__ constexpr int ring_x(int k) { return k < 2 ? 0 : ((k & 1) ? 1 : -1); }
__host__ __device__ constexpr int ring_y(int k) { return k < 2 ? ((k & 1) ? 1 : -1) : (k < 4 ? -1 : k < 6 ? 0 : 1); }

__device__ __forceinline__ uint32_t fsme_block_sad(const uint8_t* __restrict__ sf, size_t plane, int pitch, int pad,
                                                   int bxp, int byp, int vx, int vy, const uint32_t (&cfb)[4]) {
  const uint8_t* pl = sf + (size_t)(4 * (vy & 3) + (vx & 3)) * plane;
  const uint8_t* p0 = pl + (size_t)(byp + (vy >> 2) + pad) * pitch + (bxp + (vx >> 2) + pad);
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

template <int MASK>
__device__ __forceinline__ uint32_t fsme_sum(uint32_t v) {   // all-reduce inside the 16-lane half
  const unsigned half = (threadIdx.x & 16) ? 0xffff0000u : 0x0000ffffu;
  if (MASK & 1) v += __shfl_xor_sync(half, v, 1);
  if (MASK & 2) v += __shfl_xor_sync(half, v, 2);
  if (MASK & 4) v += __shfl_xor_sync(half, v, 4);
  if (MASK & 8) v += __shfl_xor_sync(half, v, 8);
  return v;
}

template <int MASK>
__device__ __forceinline__ void fsme_mode(const MeParams& P, const uint8_t* __restrict__ sf, int p, size_t o,
                                          const uint32_t* mvs_s, const uint32_t* sads_s, int bxp, int byp, int b,
                                          const uint32_t (&cfb)[4]) {
  const uint32_t mv = mvs_s[p];
  const int cx = 4 * (int)(int16_t)(mv & 0xffffu), cy = 4 * (int)(int16_t)(mv >> 16);
  uint32_t best = sads_s[p];                  // centre cost = the ME SAD (phase 0 = integer samples)
  int bvx = cx, bvy = cy;
#pragma unroll
  for (int stage = 0; stage < 2; ++stage) {
    const int ox = bvx, oy = bvy;             // half: around c; quarter: around the best half position
    uint32_t sad[8];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      sad[k] = fsme_block_sad(sf, P.sf_plane, P.sf_pitch, P.sf_pad, bxp, byp, ox + (ring_x(k) << (1 - stage)),
                              oy + (ring_y(k) << (1 - stage)), cfb);
#pragma unroll
    for (int k = 0; k < 8; ++k) {             // spiral order, strict < (G14)
      const uint32_t t = fsme_sum<MASK>(sad[k]);
      if (t < best) { best = t; bvx = ox + (ring_x(k) << (1 - stage)); bvy = oy + (ring_y(k) << (1 - stage)); }
    }
  }
  if ((b & MASK) == 0) {                      // partition leader writes
    P.out_qmvs[o + p] = (uint32_t)(uint16_t)bvx | ((uint32_t)(uint16_t)bvy << 16);
    P.out_qsads[o + p] = (uint16_t)best;
  }
}

__device__ __forceinline__ void fused_sme(const MeParams& P, const uint32_t* cf_s, const uint32_t* win_mv,
                                          const uint32_t* win_sad, int mbx) {
  const int b = threadIdx.x & 15;
  const int bx0 = b & 1, by0 = (b >> 1) & 1, bx1 = (b >> 2) & 1, by1 = (b >> 3) & 1;
  const int bx = 2 * bx1 + bx0, by = 2 * by1 + by0;
  const int bxp = 16 * mbx + 4 * bx, byp = 16 * (P.row0 + blockIdx.y) + 4 * by;
  uint32_t cfb[4];
#pragma unroll
  for (int r = 0; r < 4; ++r) cfb[r] = cf_s[(4 * by + r) * 4 + bx];
  const int s = 2 * by1 + bx1;
  const int groups = blockDim.x >> 4;
  for (int ref = threadIdx.x >> 4; ref < P.n_rf; ref += groups) {   // whole 16-lane halves iterate together
    const uint8_t* __restrict__ sf = P.sf[ref];
    const uint32_t* mvs_s = win_mv + ref * kNPart;
    const uint32_t* sads_s = win_sad + ref * kNPart;
    const size_t o = ((size_t)(blockIdx.y * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart;
    fsme_mode<15>(P, sf, 0, o, mvs_s, sads_s, bxp, byp, b, cfb);                           // 16x16
    fsme_mode<7>(P, sf, 1 + by1, o, mvs_s, sads_s, bxp, byp, b, cfb);                      // 16x8
    fsme_mode<11>(P, sf, 3 + bx1, o, mvs_s, sads_s, bxp, byp, b, cfb);                     // 8x16
    fsme_mode<3>(P, sf, 5 + s, o, mvs_s, sads_s, bxp, byp, b, cfb);                        // 8x8
    fsme_mode<1>(P, sf, 9 + 2 * s + by0, o, mvs_s, sads_s, bxp, byp, b, cfb);              // 8x4
    fsme_mode<2>(P, sf, 17 + 2 * s + bx0, o, mvs_s, sads_s, bxp, byp, b, cfb);             // 4x8
    fsme_mode<0>(P, sf, 25 + 4 * s + 2 * by0 + bx0, o, mvs_s, sads_s, bxp, byp, b, cfb);   // 4x4
  }
}

// S_CT = compile-time SA size (0 = any even S read from P at run time);
// FUSE = also run the SME of this MB (fused_sme) after its ME;
// KSH = key shift: 16 (pure SAD) or 15 (rate term, G18: J may exceed 16 bits);
// PMV = the G21 predictor is read (always possible in the runtime-S kernel).
template <int S_CT, bool FUSE = false, int KSH = 16, bool PMV = false>
// S_CT > 0: <= 128 candidates/axis -> <= 4 warps, 4 CTAs/SM.  S_CT == 0 (runtime S,
// incl. the inclusive SA's 129 candidates -> 5 warps): same 128-register cap.
__global__ void __launch_bounds__(S_CT ? 128 : 256, S_CT ? FEVES_ME_MINB : 2) me_fsbm_kernel(const MeParams P) {
  extern __shared__ __align__(16) uint32_t smem[];
  // S = candidates per axis: sa_range (G1), or sa_range + 1 for the inclusive SA (f4);
  // candidates dx, dy in [-R, hi], hi = S - 1 - R (R - 1, or R when inclusive)
  const int S = S_CT ? S_CT : P.S;
  const int R = S_CT ? S_CT / 2 : P.R;
  const int hi = S - 1 - R;
  const int PW = me_pw(S), CSTRIDE = me_cstride(S), LX = me_lx(S), NGX = me_ngx(S);
  const int NSUB = me_nsub(S), DYL = me_dyl(S);
  uint32_t* cf_s = smem;                                  // 16 rows x 4 words
  uint32_t* win = smem + 64;                              // 4 copies x CSTRIDE words
  constexpr bool QUAD = QuadKeys<S_CT, KSH>::value;
  constexpr int NH = QUAD ? 2 : 1;                        // dy halves reduced separately
  uint32_t* red = win + 4 * CSTRIDE;                      // [nwarps][NH][41]
  uint32_t* win_mv = red + (blockDim.x >> 5) * me_red_halves(S) * kNPart;   // FUSE: [n_rf][41] MVs, then SADs
  uint32_t* win_sad = win_mv + P.n_rf * kNPart;

  const int mbx = blockIdx.x, mby = P.row0 + blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t one = (uint32_t)(P.n_rf > 0);              // == 1, opaque to the compiler (see fadd)
  const int nwarps = blockDim.x >> 5;

  // ---- lane geometry: dx column and dy sub-range ----
  const int gx = warp % NGX, wy = me_nwy(S) > 1 ? warp / NGX : 0;
  const int xi = lane % LX, sub = wy * NSUB + lane / LX;
  const int dx = min(-R + gx * LX + xi, hi);               // beyond-range lanes duplicate dx=hi
  const int off = dx + R;                                  // byte offset inside the window row
  const uint32_t* wbase = win + (off & 3) * CSTRIDE + (off >> 2);
  const int dy_begin = -R + sub * DYL;

  // ---- CF MB -> shared memory (read back as broadcast LDS.128 rows) ----
  // Small SAs (S <= 32: one RF window of few candidates per CTA, latency-bound grids) keep the
  // CF word in a register and store it after the first window's loads are issued, so the two
  // global round trips overlap instead of serialising (the S = 64 / 128 kernels are unchanged).
#ifndef FEVES_ME_LATECF_MAX
#define FEVES_ME_LATECF_MAX 32
#endif
  constexpr bool kLateCf = S_CT > 0 && S_CT <= FEVES_ME_LATECF_MAX && !FUSE;
  uint32_t cf_w[2] = {0, 0};                              // 64 words over 32 (S = 32) or 64 (S = 16) threads
  if (kLateCf) {
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const int i = threadIdx.x + j * (int)blockDim.x;
      if (i < 64) cf_w[j] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * (i & 3), 16 * mby + (i >> 2));
    }
  } else {
    for (int i = threadIdx.x; i < 64; i += blockDim.x)
      cf_s[i] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * (i & 3), 16 * mby + (i >> 2));
  }

  const int xw0 = 16 * mbx - R, yw0 = 16 * mby - R;
  constexpr int NSTG = S_CT ? me_nstage(S_CT) : 1;      // window stagings per RF (dy halves)
  const int win_rows = S_CT ? me_win_rows(S_CT) : S + 15;

  const int ref_begin = (int)blockIdx.z * P.rf_per_cta, ref_end = min(P.n_rf, ref_begin + P.rf_per_cta);
  for (int ref = ref_begin; ref < ref_end; ++ref) {
    const uint8_t* __restrict__ rf = P.rf[ref];
    // G21: the SA of this (MB, RF) is centred on the clamped predictor p (runtime-S kernel and the
    // PMV instantiations; the default compile-time kernels never see a predictor, code unchanged)
    constexpr bool kPmv = S_CT == 0 || PMV;
    int pcx = 0, pcy = 0;
    if (kPmv && P.pmv) {
      const size_t pi = ((size_t)mby * P.mb_cols + mbx) * P.rf_stride + ref;
      pcx = min(max((int)P.pmv[2 * pi], -P.max_pmv), P.max_pmv);
      pcy = min(max((int)P.pmv[2 * pi + 1], -P.max_pmv), P.max_pmv);
    }
    uint32_t M[kNPart];
#pragma unroll
    for (int p = 0; p < kNPart; ++p) M[p] = 0xffffffffu;

    // the lane's rank column (dy contiguous): with a compile-time S (a multiple of 4)
    // every chunk start dy0 + R is a multiple of 4, so a chunk's ranks are ONE LDG.128
    const uint32_t* rank_col = P.rank_tab + off * me_rank_pitch(S) + R;
    uint32_t rank_next[kMeT];
    auto load_ranks = [&](int d0) {
      if (S_CT > 0 && kMeT == 4) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(rank_col + d0));
        rank_next[0] = v.x; rank_next[1] = v.y; rank_next[2] = v.z; rank_next[3] = v.w;
      } else {
#pragma unroll
        for (int t = 0; t < kMeT; ++t) rank_next[t] = __ldg(rank_col + d0 + t);
      }
    };
    load_ranks(min(dy_begin, hi + 1 - kMeT));

#pragma unroll 1
    for (int hs = 0; hs < NSTG; ++hs) {
    const int yst = yw0 + pcy + hs * (S / NSTG);          // frame row of staged window row 0
    __syncthreads();
    // ---- a1: stage 4 byte-shifted copies of the SA window ----
    // item = (window row, 16-byte chunk k): raw words 4k..4k+4 -> words 4k..4k+3
    // of copies 0..3 (copy c word q = raw bytes [4q+c, 4q+c+4)), STS.128.
    {
      const int chunks = PW >> 2;
      const bool vec_ok = P.vec_ok && (pcx & 15) == 0;
      for (int item = threadIdx.x; item < win_rows * chunks; item += blockDim.x) {
        const int row = item / chunks, k = item - row * chunks;
        const int x = xw0 + pcx + 16 * k, y = min(max(yst + row, 0), P.H - 1);
        uint32_t w[5];
        if (vec_ok && x >= 0 && x + 20 <= P.W) {
          const uint8_t* src = rf + (size_t)y * P.W + x;
          const uint4 v = __ldg(reinterpret_cast<const uint4*>(src));
          w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
          w[4] = __ldg(reinterpret_cast<const uint32_t*>(src + 16));
        } else if (kPmv && P.vec_ok && x >= 0 && (x & ~3) + 24 <= P.W) {
          // G21: a predictor moves the window start off the 16-byte grid; the rows are still
          // aligned, so 6 aligned words + funnel shifts instead of per-byte clamped loads
          const uint32_t* src = reinterpret_cast<const uint32_t*>(rf + (size_t)y * P.W + (x & ~3));
          const uint32_t sh = 8u * (uint32_t)(x & 3);
          uint32_t a[6];
#pragma unroll
          for (int i = 0; i < 6; ++i) a[i] = __ldg(src + i);
#pragma unroll
          for (int i = 0; i < 5; ++i) w[i] = __funnelshift_r(a[i], a[i + 1], sh);
        } else {
#pragma unroll
          for (int i = 0; i < 5; ++i) w[i] = load4_clamped(rf, P.W, P.H, x + 4 * i, y);
        }
        uint32_t* dst = win + row * PW + 4 * k;
        *reinterpret_cast<uint4*>(dst) = make_uint4(w[0], w[1], w[2], w[3]);
        *reinterpret_cast<uint4*>(dst + CSTRIDE) =
            make_uint4(__byte_perm(w[0], w[1], 0x4321), __byte_perm(w[1], w[2], 0x4321),
                       __byte_perm(w[2], w[3], 0x4321), __byte_perm(w[3], w[4], 0x4321));
        *reinterpret_cast<uint4*>(dst + 2 * CSTRIDE) =
            make_uint4(__byte_perm(w[0], w[1], 0x5432), __byte_perm(w[1], w[2], 0x5432),
                       __byte_perm(w[2], w[3], 0x5432), __byte_perm(w[3], w[4], 0x5432));
        *reinterpret_cast<uint4*>(dst + 3 * CSTRIDE) =
            make_uint4(__byte_perm(w[0], w[1], 0x6543), __byte_perm(w[1], w[2], 0x6543),
                       __byte_perm(w[2], w[3], 0x6543), __byte_perm(w[3], w[4], 0x6543));
      }
    }
    if (kLateCf && ref == ref_begin) {                   // the CTA's first RF
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int i = threadIdx.x + j * (int)blockDim.x;
        if (i < 64) cf_s[i] = cf_w[j];
      }
    }
    __syncthreads();

    for (int c = hs * (DYL / NSTG); c < (hs + 1) * (DYL / NSTG); c += kMeT) {
      const int dy0 = min(dy_begin + c, hi + 1 - kMeT);   // clamped chunk: duplicates are harmless
      uint32_t rank[kMeT];
#pragma unroll
      for (int t = 0; t < kMeT; ++t) rank[t] = rank_next[t];
      {                                                   // prefetch the next chunk's ranks
        load_ranks(min(dy_begin + c + kMeT, hi + 1 - kMeT));
      }
      const uint32_t* wrow = wbase + (dy0 + R - hs * (S / NSTG)) * PW;

      uint32_t acc[kMeT][4];
      RowState st[kMeT];
      uint32_t Kp[kMeT][16];
      uint4 cfr[16];
#pragma unroll
      for (int i = 0; i < kMeT + 15; ++i) {
        if (i < 16) cfr[i] = lds128_v(cf_s + 4 * i);     // CF row i, used by RF rows i..i+3
        uint32_t w[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) w[b] = wrow[i * PW + b];
        // all SADs of this RF row first (word-major), then the keys / folds of the candidates
        // whose 4x4 block row it completes (measured 0.3% faster than candidate-major)
#pragma unroll
        for (int b = 0; b < 4; ++b)
#pragma unroll
          for (int t = 0; t < kMeT; ++t) {
            const int r = i - t;                            // CF row paired with RF row i
            if (r >= 0 && r < 16) {
              const uint32_t cw[4] = {cfr[r].x, cfr[r].y, cfr[r].z, cfr[r].w};
              acc[t][b] = vad4(cw[b], w[b], (r & 3) ? acc[t][b] : 0u);
            }
          }
#pragma unroll
        for (int t = 0; t < kMeT; ++t) {
          const int r = i - t;
          if (r >= 0 && r < 16) {
            if ((r & 3) == 3) {
              const int by = r >> 2;
              if (SumKeys<S_CT, KSH>::value) {
                if (by == 0) block_row_keys_sum<0>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 1) block_row_keys_sum<1>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 2) block_row_keys_sum<2>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 3) block_row_keys_sum<3>(acc[t], rank[t], st[t], Kp[t], one);
              } else {
                if (by == 0) block_row_keys<0, KSH>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 1) block_row_keys<1, KSH>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 2) block_row_keys<2, KSH>(acc[t], rank[t], st[t], Kp[t], one);
                if (by == 3) block_row_keys<3, KSH>(acc[t], rank[t], st[t], Kp[t], one);
              }
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

    if (QUAD && hs == 0) {                                // end of the dy < 0 quadrant half
#pragma unroll
      for (int p = 0; p < kNPart; ++p) {
        const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
        if (lane == 0) red[(warp * NH) * kNPart + p] = v;
        M[p] = 0xffffffffu;
      }
    }
    }   // hs

    // ---- a4: warp min (CREDUX), then CTA min through shared memory ----
#pragma unroll
    for (int p = 0; p < kNPart; ++p) {
      const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
      if (lane == 0) red[(warp * NH + NH - 1) * kNPart + p] = v;
    }
    __syncthreads();
    for (int p = threadIdx.x; p < kNPart; p += blockDim.x) {
      uint32_t k, rk, sad;
      if (QUAD) {                                            // (SAD, global dense rank), 30 bits
        k = 0xffffffffu;
        for (int w = 0; w < nwarps; ++w)
          for (int hf = 0; hf < 2; ++hf) {
            const uint32_t v = red[(w * 2 + hf) * kNPart + p];
            const int q = 2 * hf + (w >= nwarps / 2 ? 1 : 0);   // quadrant: dy half, dx half
            const uint32_t g = __ldg(P.glob_tab + q * 4096 + ((v & 0xffffu) >> part_log2n(p)));
            k = min(k, ((v >> 16) << 14) | g);
          }
        rk = k & 0x3fffu;
        sad = k >> 14;
      } else {
        k = red[p];
        for (int w = 1; w < nwarps; ++w) k = min(k, red[w * kNPart + p]);
        rk = SumKeys<S_CT, KSH>::value ? (k & 0xffffu) >> part_log2n(p) : k & ((1u << KSH) - 1u);
        sad = k >> KSH;                                      // J = SAD + lambda*R(mv) (G18)
      }
      uint32_t mv = __ldg(P.inv_tab + rk);                   // SA offset (dx, dy)
      if (KSH != 16)                                         // rate of the offset = R(mv - p) (G21)
        sad -= (uint32_t)(P.lambda * (se_bits(4 * (int)(int16_t)(mv & 0xffffu)) + se_bits(4 * (int)(int16_t)(mv >> 16))));
      if (kPmv && P.pmv)                                     // mv = p + offset (G21)
        mv = (uint32_t)(uint16_t)((int)(int16_t)(mv & 0xffffu) + pcx) |
             ((uint32_t)(uint16_t)((int)(int16_t)(mv >> 16) + pcy) << 16);
      const size_t o = ((size_t)(blockIdx.y * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
      if (P.out_mvs) {
        reinterpret_cast<uint32_t*>(P.out_mvs)[o] = mv;
        P.out_sads[o] = (uint16_t)sad;
      }
      if (FUSE) {
        win_mv[ref * kNPart + p] = mv;
        win_sad[ref * kNPart + p] = sad;
      }
    }
  }
  if (FUSE) {
    __syncthreads();
    fused_sme(P, cf_s, win_mv, win_sad, mbx);
  }
}

}  // namespace feves
