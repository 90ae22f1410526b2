// sme_refine.cuh -- SME: sub-pixel refinement of the ME MVs.
//
// P:6: "By relying on the MVs from the ME and the SFs from the INT, the
// Sub-Pixel Motion Estimation (SME) is applied to further refine the MVs";
// "the MVs from ME define the initial search point for the SME".
// Algorithm (O3, G12-G14): centre c = 4*mv (cost = ME SAD); half
// stage: the 8 ring-1 neighbours c + 2*s_k in spiral order, update on strict
// <; quarter stage: the 8 neighbours of the best half position, strict <.
//
// Mapping (L1-sector bound kernel): one warp = 8 horizontally
// adjacent MBs of one RF x 4 lanes; lane (g, bx) owns the 4-pixel column
// strip bx of MB g (its four 4x4 blocks by = 0..3); the lane refines the
// partitions of its strip one after the other, loading only that partition's
// CF rows (80 registers -> 24 resident warps per SM for a latency-bound kernel).
// For one candidate, every LDG of the warp reads one row of 8 x 16 contiguous
// bytes of one SF phase plane when the MBs' MVs agree (the common case), so a
// request touches ~5 sectors instead of 16.  A partition's SAD = sum over its
// blocks: inside the lane over by, across lanes by xor-shuffles over bx bits;
// every lane of a partition then holds the same (best, bestv) -- no divergence.
#pragma once
#include "common.cuh"
#include "me_fsbm.cuh"   // se_bits (G18)

namespace feves {

struct SmeParams {
  const uint8_t* cf;
  const uint8_t* sf[kMaxRf];
  const uint32_t* in_mvs;     // int16 pairs as u32
  const uint16_t* in_sads;    // may be null
  uint32_t* out_qmvs;
  uint16_t* out_sads;
  int W, H, n_rf, rf_stride, mb_cols, row0, n_rows;   // n_rf RFs refined, rf_stride = layout
  int groups;                                         // ceil(mb_cols / 8)
  int pad, pitch;
  size_t plane;
  int lambda;                                         // G18 rate term (0 = pure SAD, G13)
  const int16_t* pmv;                                 // G21 predictor [frame MB][rf_stride][2] or null
  int max_pmv;
  int fence;                                          // outputs are peer memory (me_ipc_open): system fence at exit
  int cf_vec;                                         // W % 4 == 0 and cf 4-byte aligned: CF rows as aligned words
  uint32_t k_hi;                                      // = kAvgHi (vavg4)
  int split;                                          // grid.y = 16 (mode, partition group) tasks instead of 7 modes
};

// ring-1 spiral order s_k (G12/G14), compile-time so unrolled loops fold it
__device__ constexpr int8_t c_ring1[8][2] = {{0, -1}, {0, 1}, {-1, -1}, {1, -1}, {-1, 0}, {1, 0}, {-1, 1}, {1, 1}};

// SAD of this lane's 4x4 block (rows ys..ys+3 of the strip) vs SF samples at quarter offset v
__device__ __forceinline__ uint32_t strip_block_sad(const uint8_t* __restrict__ sf, size_t plane, int pitch, int pad,
                                                    int xs, int ys, int vx, int vy, const uint32_t* cfr) {
  const uint8_t* pl = sf + (size_t)(4 * (vy & 3) + (vx & 3)) * plane;
  const uint8_t* p0 = pl + (size_t)(ys + (vy >> 2) + pad) * pitch + (xs + (vx >> 2) + pad);
  const uintptr_t a = reinterpret_cast<uintptr_t>(p0);
  const uint32_t* w = reinterpret_cast<const uint32_t*>(a & ~uintptr_t(3));
  const uint32_t sh = 8u * (uint32_t)(a & 3);
  const int wp = pitch >> 2;
  uint32_t s = 0;
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const uint32_t lo = __ldg(w + r * wp), hi = __ldg(w + r * wp + 1);
    s = vad4(cfr[r], __funnelshift_r(lo, hi, sh), s);
  }
  return s;
}

// G20: SATD of one 4x4 block = (sum |H D H^T| + 1) >> 1, D = CF - prediction,
// rows given as packed byte words.  Butterflies (the abs-sum does not depend on
// the Hadamard row order).
__device__ __forceinline__ uint32_t satd4(const uint32_t* cfr, const uint32_t* smp) {
  int t[4][4];
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    int d[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) d[i] = (int)((cfr[r] >> (8 * i)) & 0xffu) - (int)((smp[r] >> (8 * i)) & 0xffu);
    const int s01 = d[0] + d[1], d01 = d[0] - d[1], s23 = d[2] + d[3], d23 = d[2] - d[3];
    t[r][0] = s01 + s23; t[r][1] = s01 - s23; t[r][2] = d01 - d23; t[r][3] = d01 + d23;
  }
  int sum = 0;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const int s01 = t[0][c] + t[1][c], d01 = t[0][c] - t[1][c], s23 = t[2][c] + t[3][c], d23 = t[2][c] - t[3][c];
    sum += abs(s01 + s23) + abs(s01 - s23) + abs(d01 - d23) + abs(d01 + d23);
  }
  return (uint32_t)((sum + 1) >> 1);
}

// SATD of this lane's 4x4 block vs SF samples at quarter offset v (loads as strip_block_sad)
__device__ __forceinline__ uint32_t strip_block_satd(const uint8_t* __restrict__ sf, size_t plane, int pitch, int pad,
                                                     int xs, int ys, int vx, int vy, const uint32_t* cfr) {
  const uint8_t* pl = sf + (size_t)(4 * (vy & 3) + (vx & 3)) * plane;
  const uint8_t* p0 = pl + (size_t)(ys + (vy >> 2) + pad) * pitch + (xs + (vx >> 2) + pad);
  const uintptr_t a = reinterpret_cast<uintptr_t>(p0);
  const uint32_t* w = reinterpret_cast<const uint32_t*>(a & ~uintptr_t(3));
  const uint32_t sh = 8u * (uint32_t)(a & 3);
  const int wp = pitch >> 2;
  uint32_t smp[4];
#pragma unroll
  for (int r = 0; r < 4; ++r) smp[r] = __funnelshift_r(__ldg(w + r * wp), __ldg(w + r * wp + 1), sh);
  return satd4(cfr, smp);
}

template <bool SATD>
__device__ __forceinline__ uint32_t strip_block_dist(const uint8_t* __restrict__ sf, size_t plane, int pitch, int pad,
                                                     int xs, int ys, int vx, int vy, const uint32_t* cfr) {
  return SATD ? strip_block_satd(sf, plane, pitch, pad, xs, ys, vx, vy, cfr)
              : strip_block_sad(sf, plane, pitch, pad, xs, ys, vx, vy, cfr);
}

// Two aligned words holding the 5 bytes at [a, a+5): the 4-byte windows at a
// (left) and a+1 (right) are both funnel shifts of them (the right one with the
// clamped shift, 32 -> the high word).  One pair of LDG per row serves the two
// horizontally adjacent half-grid windows of the SME (same plane, columns x, x+1).
// The SF pitch and plane size are multiples of 16 bytes (G11 layout), so a
// sweep's rows share one alignment: the aligned word pointer and the byte shift
// are computed once per sweep (RowP) and each row costs 2 LDG + the funnel shifts.
// SF row word load.  FEVES_SME_L2PF = 128 / 256: the same non-coherent load with an L2
// sector-promotion hint (experiment knob; 0 = plain __ldg, the default)
#ifndef FEVES_SME_L2PF
#define FEVES_SME_L2PF 0
#endif
__device__ __forceinline__ uint32_t sf_ld(const uint32_t* p) {
#if FEVES_SME_L2PF == 128
  uint32_t v;
  asm("ld.global.nc.L2::128B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#elif FEVES_SME_L2PF == 256
  uint32_t v;
  asm("ld.global.nc.L2::256B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}
struct Win2 { uint32_t l, r; };
#ifndef FEVES_SME_OFF32
#define FEVES_SME_OFF32 1
#endif
#if FEVES_SME_OFF32
// a sweep's row pointer as a 32-bit word offset from ONE shared 64-bit base (the SF's first
// word): 2 registers per row pointer instead of 3 (the kernel is register-capped at 80)
struct RowP { const uint32_t* w0; uint32_t o, sh; };
__device__ __forceinline__ RowP rowp_at(const uint8_t* sf, size_t byte_off) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(sf);
  const uint32_t b = (uint32_t)(a & 3) + (uint32_t)byte_off;
  return {reinterpret_cast<const uint32_t*>(a & ~uintptr_t(3)), b >> 2, 8u * (b & 3)};
}
__device__ __forceinline__ Win2 ld_lr(const RowP& q, int off) {   // off = row * (pitch / 4)
  const uint32_t* p = q.w0 + (q.o + (uint32_t)off);
  const uint32_t w0 = sf_ld(p), w1 = sf_ld(p + 1);
  return {__funnelshift_r(w0, w1, q.sh), __funnelshift_rc(w0, w1, q.sh + 8u)};
}
__device__ __forceinline__ uint32_t ld_w(const RowP& q, int off) {
  const uint32_t* p = q.w0 + (q.o + (uint32_t)off);
  return __funnelshift_r(sf_ld(p), sf_ld(p + 1), q.sh);
}
#define FEVES_ROWP(sf, p) rowp_at((sf), (size_t)((p) - (sf)))
#else
struct RowP { const uint32_t* w; uint32_t sh; };
__device__ __forceinline__ RowP rowp(const uint8_t* p) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(p);
  return {reinterpret_cast<const uint32_t*>(a & ~uintptr_t(3)), 8u * (uint32_t)(a & 3)};
}
__device__ __forceinline__ Win2 ld_lr(const RowP& q, int off) {   // off = row * (pitch / 4)
  const uint32_t w0 = sf_ld(q.w + off), w1 = sf_ld(q.w + off + 1);
  return {__funnelshift_r(w0, w1, q.sh), __funnelshift_rc(w0, w1, q.sh + 8u)};
}
__device__ __forceinline__ uint32_t ld_w(const RowP& q, int off) {
  return __funnelshift_r(sf_ld(q.w + off), sf_ld(q.w + off + 1), q.sh);
}
#define FEVES_ROWP(sf, p) rowp(p)
#endif

// Half stage, SAD, one block group of HR rows (DESIGN.md §6 "row sweep"): for the
// full-pel centre (mx, my) the 8 ring candidates c + 2 s_k are windows of three
// half-sample planes at integer offsets (phase 4*yFrac + xFrac, G11):
//   (0,-1) h @ (mx, my-1)    (0,+1) h @ (mx, my)
//   (-1,-1) j @ (mx-1, my-1) (+1,-1) j @ (mx, my-1)
//   (-1,0) b @ (mx-1, my)    (+1,0) b @ (mx, my)
//   (-1,+1) j @ (mx-1, my)   (+1,+1) j @ (mx, my)
// so sweeping plane rows my-1 .. my+HR-1 once, each h / j row serves a candidate
// above (CF row r) and one below (CF row r-1), and each j / b row pair of words
// serves the left and right candidate: 6 LDG per row instead of 16.
template <int HR>
__device__ __forceinline__ void half_sad_sweep(const uint8_t* __restrict__ sf, size_t plane, int pitch,
                                               const uint8_t* base, int mx, int my, const uint32_t* cf,
                                               uint32_t (&sad)[8]) {
  // base = plane 0 at the strip's top-left integer sample (pad applied)
  const RowP ph = FEVES_ROWP(sf, base + 8 * plane + (ptrdiff_t)(my - 1) * pitch + mx);
  const RowP pj = FEVES_ROWP(sf, base + 10 * plane + (ptrdiff_t)(my - 1) * pitch + (mx - 1));
  const RowP pb = FEVES_ROWP(sf, base + 2 * plane + (ptrdiff_t)my * pitch + (mx - 1));
  const int wp = pitch >> 2;
#pragma unroll
  for (int k = 0; k < 8; ++k) sad[k] = 0;
#pragma unroll
  for (int r = 0; r <= HR; ++r) {
    const uint32_t hw = ld_w(ph, r * wp);
    const Win2 jw = ld_lr(pj, r * wp);
    if (r < HR) {
      const Win2 bw = ld_lr(pb, r * wp);
      sad[0] = vad4(cf[r], hw, sad[0]);
      sad[2] = vad4(cf[r], jw.l, sad[2]);
      sad[3] = vad4(cf[r], jw.r, sad[3]);
      sad[4] = vad4(cf[r], bw.l, sad[4]);
      sad[5] = vad4(cf[r], bw.r, sad[5]);
    }
    if (r > 0) {
      sad[1] = vad4(cf[r - 1], hw, sad[1]);
      sad[6] = vad4(cf[r - 1], jw.l, sad[6]);
      sad[7] = vad4(cf[r - 1], jw.r, sad[7]);
    }
  }
}

// the 8 quarter candidates around half-grid point H from its 3x3 half-grid
// windows hp[b][a] (rows hy-1..hy+1, columns hx-1..hx+1), O2 averaging rule
__device__ __forceinline__ uint32_t quarter_win(const uint32_t (&hp)[3][3], int k, bool mixed, uint32_t kh) {
  const int dx = k < 2 ? 0 : ((k & 1) ? 1 : -1);
  const int dy = k < 2 ? ((k & 1) ? 1 : -1) : (k < 4 ? -1 : k < 6 ? 0 : 1);
  if (dx == 0 || dy == 0) return vavg4(hp[1][1], hp[1 + dy][1 + dx], kh);
  return vavg4(mixed ? hp[1][1] : hp[1][1 + dx], mixed ? hp[1 + dy][1 + dx] : hp[1 + dy][1], kh);
}

// Quarter stage, SAD, one block group of HR rows, around half-grid point (hx, hy):
// half-grid columns hx-1 and hx+1 share a plane and are adjacent integer columns
// (one load_lr), likewise rows hy-1 and hy+1 are adjacent rows of one plane, so
// the sweep reads "outer" rows (hy+-1 parity) r = 0..HR and "middle" rows (hy
// parity) r = 0..HR-1, 4 LDG each, and CF row r uses outer r, middle r, outer r+1.
template <int HR>
__device__ __forceinline__ void quarter_sad_sweep(const uint8_t* sf, size_t plane, int pitch, const uint8_t* base,
                                                  int hx, int hy, const uint32_t* cf, uint32_t (&qs)[8], uint32_t kh) {
  const bool mixed = ((hx ^ hy) & 1) != 0;
  const int xm = hx - 1, x0 = hx, ym = hy - 1, y0 = hy;
  auto at = [&](int X, int Y) {                 // plane row pointer of half-grid point (X, Y), CF row 0
    return base + (size_t)(8 * (Y & 1) + 2 * (X & 1)) * plane + (ptrdiff_t)(Y >> 1) * pitch + (X >> 1);
  };
  const RowP o_lr = FEVES_ROWP(sf, at(xm, ym));   // outer rows, columns hx-1 / hx+1
  const RowP o_c = FEVES_ROWP(sf, at(x0, ym));    // outer rows, column hx
  const RowP m_lr = FEVES_ROWP(sf, at(xm, y0));   // middle rows
  const RowP m_c = FEVES_ROWP(sf, at(x0, y0));
  const int wp = pitch >> 2;
#pragma unroll
  for (int k = 0; k < 8; ++k) qs[k] = 0;
  uint32_t po[3], pm[3];                        // previous outer / middle windows (L, C, R)
#pragma unroll
  for (int r = 0; r <= HR; ++r) {
    const Win2 olr = ld_lr(o_lr, r * wp);
    const uint32_t oc = ld_w(o_c, r * wp);
    if (r > 0) {
      const uint32_t hp[3][3] = {{po[0], po[1], po[2]}, {pm[0], pm[1], pm[2]}, {olr.l, oc, olr.r}};
#pragma unroll
      for (int k = 0; k < 8; ++k) qs[k] = vad4(cf[r - 1], quarter_win(hp, k, mixed, kh), qs[k]);
    }
    if (r < HR) {
      const Win2 mlr = ld_lr(m_lr, r * wp);
      pm[0] = mlr.l; pm[1] = ld_w(m_c, r * wp); pm[2] = mlr.r;
      po[0] = olr.l; po[1] = oc; po[2] = olr.r;
    }
  }
}

template <int XMASK>
__device__ __forceinline__ uint32_t xsum(uint32_t v) {   // all-reduce over the bx lane bits in XMASK
  if (XMASK & 1) v += __shfl_xor_sync(0xffffffffu, v, 1);
  if (XMASK & 2) v += __shfl_xor_sync(0xffffffffu, v, 2);
  return v;
}

// partition index (G7) of block (bx, by) in each mode
template <int MODE>
__device__ __forceinline__ int mode_part(int bx, int by) {
  const int s = 2 * (by >> 1) + (bx >> 1);
  switch (MODE) {
    case 0: return 0;                                      // 16x16
    case 1: return 1 + (by >> 1);                          // 16x8
    case 2: return 3 + (bx >> 1);                          // 8x16
    case 3: return 5 + s;                                  // 8x8
    case 4: return 9 + 2 * s + (by & 1);                   // 8x4 (w8 h4)
    case 5: return 17 + 2 * s + (bx & 1);                  // 4x8 (w4 h8)
    default: return 25 + 4 * s + 2 * (by & 1) + (bx & 1);  // 4x4
  }
}

// YG = blocks of a partition along by inside the lane (1, 2, 4);
// XMASK = the bx lane bits a partition spans (0, 1, 3).
//
// Half stage: the 8 candidates c + 2 s_k are half-grid samples, read from the
// b / h / j planes (phases 2, 8, 10).  Quarter stage: the 8 neighbours of the
// best half position H are, by the interpolation rule itself (O2: every
// quarter sample is the rounded average of two half-grid samples), rounded
// averages of the 3x3 half-grid samples around H.  Those 9 windows per row come
// from the 4 planes G, b, h, j only (phases 0, 2, 8, 10), so the refinement
// touches 4 of the 16 planes (4x less L1/L2 footprint); the averages are the
// SWAR byte average, bit-identical to the quarter planes INT writes.
// Axis neighbour (dx,0) = avg(HP(0,0), HP(dx,0)), (0,dy) likewise; diagonal
// (dx,dy) = avg of the two corners of the half-grid unit square that have one
// odd coordinate: (0,0) & (dx,dy) if H has mixed parity, else (dx,0) & (0,dy).
// RD = rate term (G18) compiled in; SATD = Hadamard distortion (G20) instead of SAD
template <int MODE, int YG, int XMASK, bool RD, bool SATD>
__device__ __forceinline__ void refine_mode(const SmeParams& P, const uint8_t* __restrict__ sf, size_t o, int bx,
                                            int xs, int ys0, bool writer, int qpx, int qpy, int g0 = 0, int g1 = 4) {
  constexpr int NG = 4 / YG;           // partitions (block groups) inside this lane's strip
  g1 = min(g1, NG);                    // this warp refines groups [g0, g1) (all NG, or one: P.split)
  // The groups are refined one after the other (latency-bound kernel: fewer live
  // registers -> more resident warps beats the ILP of refining all NG at once).
  // the next group's ME result (MV, SAD) is loaded one group ahead, so only the first
  // group pays the dependent MV -> SF-address round trip
  uint32_t mv_n = __ldg(P.in_mvs + o + mode_part<MODE>(bx, g0 * YG));
  uint32_t sad_n = (P.in_sads && !SATD) ? (uint32_t)__ldg(P.in_sads + o + mode_part<MODE>(bx, g0 * YG)) : 0u;
#pragma unroll 1
  for (int g = g0; g < g1; ++g) {
    const uint32_t mv = mv_n, sad_me = sad_n;
    if (g + 1 < g1) {
      const int pn = mode_part<MODE>(bx, (g + 1) * YG);
      mv_n = __ldg(P.in_mvs + o + pn);
      if (P.in_sads && !SATD) sad_n = __ldg(P.in_sads + o + pn);
    }
    const int yg = ys0 + 4 * g * YG;   // first frame row of this group
    uint32_t cf[4 * YG];               // this group's CF strip rows
    if (P.cf_vec && xs + 3 < P.W && yg + 4 * YG <= P.H) {        // inside the frame: aligned words
      const uint32_t* c0 = reinterpret_cast<const uint32_t*>(P.cf + (size_t)yg * P.W + xs);
#pragma unroll
      for (int r = 0; r < 4 * YG; ++r) cf[r] = __ldg(c0 + r * (P.W >> 2));
    } else {                                                      // clamped (G5, G6)
#pragma unroll
      for (int r = 0; r < 4 * YG; ++r) cf[r] = load4_clamped(P.cf, P.W, P.H, xs, yg + r);
    }
    const int p = mode_part<MODE>(bx, g * YG);
    int bvx = 4 * (int)(int16_t)(mv & 0xffffu);
    int bvy = 4 * (int)(int16_t)(mv >> 16);
    uint32_t best;
    if (P.in_sads && !SATD) {
      best = sad_me;
    } else {
      uint32_t s = 0;
#pragma unroll
      for (int j = 0; j < YG; ++j)
        s += strip_block_dist<SATD>(sf, P.plane, P.pitch, P.pad, xs, yg + 4 * j, bvx, bvy, cf + 4 * j);
      best = xsum<XMASK>(s);
    }
    if (RD) best += P.lambda * (se_bits(bvx - qpx) + se_bits(bvy - qpy));   // J at the centre
    // ---- half stage ----
    {
      const int ox = bvx, oy = bvy;
      uint32_t sad[8];
      if (!SATD) {                                    // SAD: one row sweep
        half_sad_sweep<4 * YG>(sf, P.plane, P.pitch, sf + (size_t)(yg + P.pad) * P.pitch + (xs + P.pad), ox >> 2,
                               oy >> 2, cf, sad);
      } else {                                        // SATD: whole 4x4 blocks per candidate
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          uint32_t t = 0;
#pragma unroll
          for (int j = 0; j < YG; ++j)
            t += strip_block_dist<SATD>(sf, P.plane, P.pitch, P.pad, xs, yg + 4 * j, ox + 2 * c_ring1[k][0],
                                        oy + 2 * c_ring1[k][1], cf + 4 * j);
          sad[k] = t;
        }
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {                 // spiral order, strict < (G14)
        const int vx = ox + 2 * c_ring1[k][0], vy = oy + 2 * c_ring1[k][1];
        uint32_t t = xsum<XMASK>(sad[k]);
        if (RD) t += P.lambda * (se_bits(vx - qpx) + se_bits(vy - qpy));
        if (t < best) { best = t; bvx = vx; bvy = vy; }
      }
    }
    // ---- quarter stage from the 3x3 half-grid windows around the best half position ----
    {
      const int hx = bvx >> 1, hy = bvy >> 1;          // half-grid coordinates (bvx, bvy even)
      uint32_t qs[8];
      if (!SATD) {                                     // SAD: one row sweep
        quarter_sad_sweep<4 * YG>(sf, P.plane, P.pitch, sf + (size_t)(yg + P.pad) * P.pitch + (xs + P.pad), hx, hy, cf, qs,
                                  P.k_hi);
      } else {                                         // SATD: whole 4x4 blocks, one candidate at a time
        const bool mixed = ((hx ^ hy) & 1) != 0;
        int off[3][3];                                 // window offsets from the strip's row base
#pragma unroll
        for (int b = 0; b < 3; ++b)
#pragma unroll
          for (int a = 0; a < 3; ++a)
            off[b][a] = (8 * ((hy + b - 1) & 1) + 2 * ((hx + a - 1) & 1)) * (int)P.plane +
                        ((hy + b - 1) >> 1) * P.pitch + ((hx + a - 1) >> 1);
#pragma unroll
        for (int k = 0; k < 8; ++k) qs[k] = 0;
        const uint8_t* rowp = sf + (size_t)(yg + P.pad) * P.pitch + (xs + P.pad);
#pragma unroll 1
        for (int jb = 0; jb < YG; ++jb, rowp += 4 * P.pitch) {
#pragma unroll 1
          for (int k = 0; k < 8; ++k) {
            const int dx = c_ring1[k][0], dy = c_ring1[k][1];
            // the two half-grid windows this quarter candidate averages (O2 rule, see above)
            int b0, a0, b1, a1;
            if (dx == 0 || dy == 0) { b0 = 1; a0 = 1; b1 = 1 + dy; a1 = 1 + dx; }
            else if (mixed) { b0 = 1; a0 = 1; b1 = 1 + dy; a1 = 1 + dx; }
            else { b0 = 1; a0 = 1 + dx; b1 = 1 + dy; a1 = 1; }
            uint32_t smp[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
              const uint8_t* rp = rowp + r * P.pitch;
              const uintptr_t e0 = reinterpret_cast<uintptr_t>(rp + off[b0][a0]);
              const uintptr_t e1 = reinterpret_cast<uintptr_t>(rp + off[b1][a1]);
              const uint32_t* w0 = reinterpret_cast<const uint32_t*>(e0 & ~uintptr_t(3));
              const uint32_t* w1 = reinterpret_cast<const uint32_t*>(e1 & ~uintptr_t(3));
              smp[r] = vavg4(__funnelshift_r(__ldg(w0), __ldg(w0 + 1), 8u * (uint32_t)(e0 & 3)),
                             __funnelshift_r(__ldg(w1), __ldg(w1 + 1), 8u * (uint32_t)(e1 & 3)), P.k_hi);
            }
            qs[k] += satd4(cf + 4 * jb, smp);
          }
        }
      }
      const int ox = bvx, oy = bvy;
#pragma unroll
      for (int k = 0; k < 8; ++k) {             // spiral order, strict < (G14)
        const int vx = ox + c_ring1[k][0], vy = oy + c_ring1[k][1];
        uint32_t t = xsum<XMASK>(qs[k]);
        if (RD) t += P.lambda * (se_bits(vx - qpx) + se_bits(vy - qpy));
        if (t < best) { best = t; bvx = vx; bvy = vy; }
      }
    }
    if (writer && (bx & XMASK) == 0) {     // partition leader lane writes
      P.out_qmvs[o + p] = (uint32_t)(uint16_t)bvx | ((uint32_t)(uint16_t)bvy << 16);
      const uint32_t d = best - (RD ? P.lambda * (se_bits(bvx - qpx) + se_bits(bvy - qpy)) : 0);
      P.out_sads[o + p] = (uint16_t)min(d, 65535u);        // SATD can exceed 16 bits (G20)
    }
  }
}

#ifndef FEVES_SME_MINB
#define FEVES_SME_MINB 5   // 96 registers, 5 CTAs x 4 warps per SM; with 32-bit row offsets (FEVES_SME_OFF32) 8 B of stack, 1 spill + 3 reloads per partition group outside the sweeps (was 72 B / 56 sites at 80 registers); 4 (128 registers): none, 147.5 vs 145.4 us; 5 / 6: 145.4 us; with the longest-first order 6 (80 registers, 16 B stack, 10 spill sites) 139.7 vs 141.4 us -- kept 5 (spill-free sweeps)
#endif
template <bool RD, bool SATD>
__global__ void __launch_bounds__(128, FEVES_SME_MINB) sme_refine_kernel(const SmeParams P) {
  const int warp_id = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int n_warps = P.n_rf * P.n_rows * P.groups;
  if (warp_id >= n_warps) return;                    // whole warps exit together
  const int lane = threadIdx.x & 31;
  const int gi = warp_id % P.groups;
  const int rem = warp_id / P.groups;
  const int mrow = rem % P.n_rows, ref = rem / P.n_rows;
  const int bx = lane & 3;
  const int mbx_raw = 8 * gi + (lane >> 2);
  const bool writer = mbx_raw < P.mb_cols;
  const int mbx = min(mbx_raw, P.mb_cols - 1);       // surplus lanes duplicate the last MB
  const int mby = P.row0 + mrow;
  const int xs = 16 * mbx + 4 * bx, ys0 = 16 * mby;
  const uint8_t* __restrict__ sf = P.sf[ref];
  const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart;
  int qpx = 0, qpy = 0;                              // G21: rate against 4p (RD only)
  if (RD && P.pmv) {
    const size_t pi = ((size_t)mby * P.mb_cols + mbx) * P.rf_stride + ref;
    qpx = 4 * min(max((int)P.pmv[2 * pi], -P.max_pmv), P.max_pmv);
    qpy = 4 * min(max((int)P.pmv[2 * pi + 1], -P.max_pmv), P.max_pmv);
  }
  // one mode per warp: 7x the independent warps (the kernel is latency-bound); with P.split one
  // partition group per warp (16 tasks: modes with 1, 2, 1, 2, 4, 2, 4 groups), for grids too small
  // to fill the GPU with 7 (a narrow MB-row stripe)
#ifndef FEVES_SME_LPT
#define FEVES_SME_LPT 1   // measured 140.4 vs 146.8 us at 1080p S64 4 RF (the long warps no longer form the tail)
#endif
  // FEVES_SME_LPT: the modes with the most partition groups per warp (4x4, 8x4: four dependent
  // MV -> sweep chains) are dispatched first, the single-group modes last
  int mode = FEVES_SME_LPT ? (0x0213546 >> (4 * (int)blockIdx.y)) & 15 : (int)blockIdx.y, g0 = 0, g1 = 4;
  if (P.split == 3) {                 // 9 tasks: the 4-group modes as two warps of 2 groups, longest first
    const int y = blockIdx.y;         // (6: 0-1), (6: 2-3), (4: 0-1), (4: 2-3), 5, 3, 1, 2, 0
    mode = y < 2 ? 6 : y < 4 ? 4 : (0x021350000 >> (4 * y)) & 15;
    g0 = y < 4 ? 2 * (y & 1) : 0;
    g1 = y < 4 ? g0 + 2 : 4;
  } else if (P.split) {
    const int y = blockIdx.y;
    mode = y < 1 ? 0 : y < 3 ? 1 : y < 4 ? 2 : y < 6 ? 3 : y < 10 ? 4 : y < 12 ? 5 : 6;
    g0 = y - (mode == 0 ? 0 : mode == 1 ? 1 : mode == 2 ? 3 : mode == 3 ? 4 : mode == 4 ? 6 : mode == 5 ? 10 : 12);
    g1 = g0 + 1;
  }
  switch (mode) {
    case 0: refine_mode<0, 4, 3, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 16x16
    case 1: refine_mode<1, 2, 3, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 16x8
    case 2: refine_mode<2, 4, 1, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 8x16
    case 3: refine_mode<3, 2, 1, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 8x8
    case 4: refine_mode<4, 1, 1, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 8x4
    case 5: refine_mode<5, 2, 0, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;   // 4x8
    default: refine_mode<6, 1, 0, RD, SATD>(P, sf, o, bx, xs, ys0, writer, qpx, qpy, g0, g1); break;  // 4x4
  }
  if (P.fence) __threadfence_system();   // stores to another GPU's buffer are performed before the kernel ends
}

}  // namespace feves
