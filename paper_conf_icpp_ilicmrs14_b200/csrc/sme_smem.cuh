// sme_smem.cuh -- SME with the sub-pel windows staged in shared memory.
//
// Same algorithm as sme_refine.cuh (O3, G12-G14; P:6 "the Sub-Pixel Motion Estimation
// (SME) is applied to further refine the MVs", "the MVs from ME define the initial
// search point for the SME"): centre c = 4*mv with the ME SAD as its cost, the 8 half-pel
// neighbours c + 2 s_k, then the 8 quarter-pel neighbours of the best half position, strict
// < in ring-1 spiral order; quarter samples as rounded averages of the half-grid planes
// G, b, h, j (bit-identical to the quarter planes INT writes).
//
// Data path.  The global-load kernel (sme_refine.cuh) is bound by L1 wavefronts: each
// 4-byte window row is two scattered LDG.32, and a warp (8 MBs x 4 strips) touches one
// line per MB when the MBs' MVs differ.  Here one CTA owns one group of 8 horizontally
// adjacent MBs of one RF and all 7 modes (7 warps, the same lane mapping as the global
// kernel: warp = mode, lane = (MB, 4-pixel strip)).  The CTA reads the 8 x 41 ME results,
// reduces the bounding box of every partition's sub-pel footprint (integer columns
// [x+mvx-1, x+mvx+w+1), rows [y+mvy-1, y+mvy+h+1)), copies that box of the planes G, b, h,
// j into shared memory with 16-byte cp.async (coalesced, no register round trip), and the
// row sweeps then read it with LDS (2 per 4-byte window + a funnel shift, 32-bit
// addressing).  Neighbouring MBs' boxes overlap, so a group stages far less than 8 single
// MBs would (~45 KB at 1080p S64 on the bench content).  A group whose box exceeds the
// region is appended to an overflow list and refined by the global-load code afterwards.
#pragma once
#include "common.cuh"
#include "me_fsbm.cuh"      // se_bits (G18)
#include "sme_refine.cuh"   // SmeParams, quarter_win, refine_mode (overflow groups)

namespace feves {


#ifndef FEVES_SME2_MB
#define FEVES_SME2_MB 8           // MBs per CTA group (8; 4 measured slower: 26% of the 4-MB boxes overflow 32 KB)
#endif
#ifndef FEVES_SME2_REGION   // staged bytes per CTA (4 planes); larger boxes -> overflow list
#define FEVES_SME2_REGION (FEVES_SME2_MB == 4 ? 32 * 1024 : 68 * 1024)
#endif
#ifndef FEVES_SME2_PITCH    // staged row pitch alignment in bytes (128: vertical MV differences keep the banks)
#define FEVES_SME2_PITCH 16
#endif
#ifndef FEVES_SME2_MINB
#define FEVES_SME2_MINB (FEVES_SME2_MB == 4 ? 6 : 3)
#endif
constexpr int kSme2Mb = FEVES_SME2_MB;
constexpr int kSme2Lpm = 4 * kSme2Mb;                  // lanes per mode: (MB, 4-pixel strip)
constexpr int kSme2Threads = kSme2Mb == 8 ? 7 * 32 : 4 * 32;   // 7 modes (+ 1 idle half-warp at 4 MBs)
constexpr int kSme2Head = (kSme2Mb * (256 + 41 * 4 + 41 * 2) + 32 + 127) & ~127;   // CF, MVs, SADs, box + mbarrier (the
                                                                                   // staged region after it: 16-B aligned for TMA)
constexpr int kSme2Smem = kSme2Head + FEVES_SME2_REGION + 16;      // + slack: a row's 2nd word
// mode of a lane group: with 4-MB groups two modes share a warp, paired by partition height so
// both halves run the same number of rows per group (m0|m2: 16, m1|m3: 8, m4|m6: 4, m5|-: 8)
__device__ __forceinline__ int sme2_mode(int tid) {
  if (kSme2Mb == 8) return tid >> 5;
  const int h = tid >> 4;                                  // half-warp 0..7 -> 0, 2, 1, 3, 4, 6, 5, 7
  return (h & ~3) | ((h & 1) << 1) | ((h >> 1) & 1);
}

__host__ __device__ constexpr int part_ox(int p) {
  return p < 3 ? 0 : p < 5 ? 8 * (p - 3) : p < 9 ? 8 * ((p - 5) & 1)
       : p < 17 ? 8 * (((p - 9) >> 1) & 1) : p < 25 ? 8 * (((p - 17) >> 1) & 1) + 4 * ((p - 17) & 1)
       : 8 * (((p - 25) >> 2) & 1) + 4 * ((p - 25) & 1);
}
__host__ __device__ constexpr int part_oy(int p) {
  return p == 0 ? 0 : p < 3 ? 8 * (p - 1) : p < 5 ? 0 : p < 9 ? 8 * ((p - 5) >> 1)
       : p < 17 ? 8 * ((p - 9) >> 2) + 4 * ((p - 9) & 1) : p < 25 ? 8 * ((p - 17) >> 2)
       : 8 * ((p - 25) >> 3) + 4 * (((p - 25) >> 1) & 1);
}
__host__ __device__ constexpr int part_w(int p) { return p < 3 ? 16 : p < 17 ? 8 : 4; }
__host__ __device__ constexpr int part_h(int p) {
  return p < 1 ? 16 : p < 3 ? 8 : p < 5 ? 16 : p < 9 ? 8 : p < 17 ? 4 : p < 25 ? 8 : 4;
}

__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v)); }
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src));
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// a window row in shared memory: aligned word address + byte shift (constant over a sweep)
struct SRow { uint32_t a, sh; };
__device__ __forceinline__ SRow srow(uint32_t byte_addr) { return {byte_addr & ~3u, 8u * (byte_addr & 3u)}; }
__device__ __forceinline__ uint32_t s_w(const SRow& q, uint32_t off) {
  return __funnelshift_r(lds32(q.a + off), lds32(q.a + off + 4), q.sh);
}
__device__ __forceinline__ Win2 s_lr(const SRow& q, uint32_t off) {
  const uint32_t w0 = lds32(q.a + off), w1 = lds32(q.a + off + 4);
  return {__funnelshift_r(w0, w1, q.sh), __funnelshift_rc(w0, w1, q.sh + 8u)};
}

// The staged box: plane k (0 G, 1 b, 2 h, 3 j) at s_reg + k * pstride, integer position
// (X, Y) (frame coordinates) at row Y - ylo, byte X + pad - X0.
struct Box {
  uint32_t s_reg, pstride, wb;
  int ylo, xoff;   // xoff = pad - X0
  __device__ __forceinline__ uint32_t at(int k, int X, int Y) const {
    return s_reg + (uint32_t)k * pstride + (uint32_t)((Y - ylo) * (int)wb + X + xoff);
  }
};

// partition index (G7) of strip bx, block row by in mode m (as mode_part<MODE>; m is
// warp-uniform, so the switch does not diverge)
__device__ __forceinline__ int mode_part_rt(int m, int bx, int by) {
  const int s = 2 * (by >> 1) + (bx >> 1);
  switch (m) {
    case 0: return 0;
    case 1: return 1 + (by >> 1);
    case 2: return 3 + (bx >> 1);
    case 3: return 5 + s;
    case 4: return 9 + 2 * s + (by & 1);
    case 5: return 17 + 2 * s + (bx & 1);
    default: return 25 + 4 * s + 2 * (by & 1) + (bx & 1);
  }
}

// The 8 ring candidates' partition costs t_k (spiral order k, G14) in ONE pass: key = t_k * 8 + k,
// min over the 8 keys (3-input mins), and an update of (best, bvx, bvy) iff min t < best -- the
// same result as the ordered strict-< scan (the first of equal minima wins).  The 8 strip sums
// are xor-shuffled as 4 packed 16-bit pairs (a strip partial SAD <= 16 rows x 4 px x 255 = 16320,
// a partition sum <= 65280: no carry between the halves).  step = 2 (half stage) or 1 (quarter).
template <bool RD>
__device__ __forceinline__ void ring_update(const uint32_t (&v)[8], int xm, int step, int ox, int oy, int lambda,
                                            int qpx, int qpy, uint32_t& best, int& bvx, int& bvy) {
  uint32_t key[8];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    uint32_t pk = v[2 * i] | (v[2 * i + 1] << 16);
    const uint32_t a = __shfl_xor_sync(0xffffffffu, pk, 1);
    pk += a & (0u - (uint32_t)(xm & 1));
    const uint32_t b = __shfl_xor_sync(0xffffffffu, pk, 2);
    pk += b & (0u - (uint32_t)((xm >> 1) & 1));
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int k = 2 * i + h;
      uint32_t t = h ? (pk >> 16) : (pk & 0xffffu);
      if (RD) t += lambda * (se_bits(ox + step * c_ring1[k][0] - qpx) + se_bits(oy + step * c_ring1[k][1] - qpy));
      key[k] = t * 8u + (uint32_t)k;
    }
  }
  const uint32_t m = min(min(min(key[0], key[1]), min(key[2], key[3])), min(min(key[4], key[5]), min(key[6], key[7])));
  if ((m >> 3) < best) {
    const int k = (int)(m & 7u);
    best = m >> 3;
    bvx = ox + step * ((int)((0x8885u >> (2 * k)) & 3u) - 1);   // ring-1 dx + 1 = 1,1,0,2,0,2,0,2
    bvy = oy + step * ((int)((0xA508u >> (2 * k)) & 3u) - 1);   // ring-1 dy + 1 = 0,2,0,0,1,1,2,2
  }
}

// TMA bulk copy global -> shared (16-byte aligned, size a multiple of 16), completing on an
// mbarrier (transaction bytes), and the mbarrier helpers
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar), "r"(phase) : "memory");
}

// One mode (warp-uniform m) of the staged CTA: the same arithmetic as refine_mode (SAD, the
// ME SADs as centre costs), ONE code body for all 7 modes with run-time partition height HR
// (so the 7 warps of a CTA share their instructions: fully unrolled per-mode bodies thrash
// the instruction cache, measured 71% "no instruction" stalls).  The sweeps walk CF rows
// c = 0 .. HR-1 four at a time, carrying the previous plane row:
//   half:    c uses h / j plane rows c (above: k = 0, 2, 3) and c + 1 (below: k = 1, 6, 7),
//            b row c (k = 4, 5)                         [plane rows my-1+q, b: my+q]
//   quarter: c uses the outer half-grid rows c, c + 1 and the middle row c (3x3 around H).
template <bool RD>
__device__ __forceinline__ void refine_mode_s(const SmeParams& P, const Box& B, int m, uint32_t s_cf, uint32_t s_mv,
                                              uint32_t s_sad, int g, int bx, int xs, int ys0, bool writer,
                                              size_t o, int qpx, int qpy) {
  const int YG = (m == 0 || m == 2) ? 4 : (m == 4 || m == 6) ? 1 : 2;   // 4x4 blocks per partition along by
  const int xm = (m <= 1) ? 3 : (m <= 4) ? 1 : 0;                        // strip bits a partition spans
  const int HR = 4 * YG, NG = 4 / YG;
  const uint32_t kh = P.k_hi;
#pragma unroll 1
  for (int gi = 0; gi < NG; ++gi) {
    const int p = mode_part_rt(m, bx, gi * YG);
    const uint32_t mv = lds32(s_mv + 4 * (g * kNPart + p));
    unsigned short sd;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(sd) : "r"(s_sad + 2 * (g * kNPart + p)));
    const int yl = 4 * gi * YG, yg = ys0 + yl;
    const uint32_t cfa = s_cf + 256 * g + 16 * yl + 4 * bx;   // CF strip row yl, +16 per row
    int bvx = 4 * (int)(int16_t)(mv & 0xffffu), bvy = 4 * (int)(int16_t)(mv >> 16);
    uint32_t best = sd;
    if (RD) best += P.lambda * (se_bits(bvx - qpx) + se_bits(bvy - qpy));
    // ---- half stage ----
    {
      const int mx = bvx >> 2, my = bvy >> 2;
      const SRow ph = srow(B.at(2, xs + mx, yg + my - 1));
      const SRow pj = srow(B.at(3, xs + mx - 1, yg + my - 1));
      const SRow pb = srow(B.at(1, xs + mx - 1, yg + my));
      uint32_t sad[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) sad[k] = 0;
      uint32_t hw = s_w(ph, 0);
      Win2 jw = s_lr(pj, 0);
#pragma unroll 1
      for (int c0 = 0; c0 < HR; c0 += 4) {
#pragma unroll
        for (int cc = 0; cc < 4; ++cc) {
          const int c = c0 + cc;
          const uint32_t off = (uint32_t)c * B.wb;
          const uint32_t cf = lds32(cfa + 16 * c);
          const uint32_t hn = s_w(ph, off + B.wb);
          const Win2 jn = s_lr(pj, off + B.wb);
          const Win2 bw = s_lr(pb, off);
          sad[0] = vad4(cf, hw, sad[0]);
          sad[2] = vad4(cf, jw.l, sad[2]);
          sad[3] = vad4(cf, jw.r, sad[3]);
          sad[4] = vad4(cf, bw.l, sad[4]);
          sad[5] = vad4(cf, bw.r, sad[5]);
          sad[1] = vad4(cf, hn, sad[1]);
          sad[6] = vad4(cf, jn.l, sad[6]);
          sad[7] = vad4(cf, jn.r, sad[7]);
          hw = hn;
          jw = jn;
        }
      }
      ring_update<RD>(sad, xm, 2, bvx, bvy, P.lambda, qpx, qpy, best, bvx, bvy);
    }
    // ---- quarter stage around the best half position (half-grid coordinates) ----
    {
      const int hx = bvx >> 1, hy = bvy >> 1;
      const bool mixed = ((hx ^ hy) & 1) != 0;
      auto at = [&](int X, int Y) { return B.at(2 * (Y & 1) + (X & 1), xs + (X >> 1), yg + (Y >> 1)); };
      const SRow o_lr = srow(at(hx - 1, hy - 1)), o_c = srow(at(hx, hy - 1));
      const SRow m_lr = srow(at(hx - 1, hy)), m_c = srow(at(hx, hy));
      uint32_t qs[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) qs[k] = 0;
      Win2 ow = s_lr(o_lr, 0);
      uint32_t oc = s_w(o_c, 0);
#pragma unroll 1
      for (int c0 = 0; c0 < HR; c0 += 4) {
#pragma unroll
        for (int cc = 0; cc < 4; ++cc) {
          const int c = c0 + cc;
          const uint32_t off = (uint32_t)c * B.wb;
          const uint32_t cf = lds32(cfa + 16 * c);
          const Win2 on = s_lr(o_lr, off + B.wb);
          const uint32_t ocn = s_w(o_c, off + B.wb);
          const Win2 mw = s_lr(m_lr, off);
          const uint32_t mc = s_w(m_c, off);
          const uint32_t hp[3][3] = {{ow.l, oc, ow.r}, {mw.l, mc, mw.r}, {on.l, ocn, on.r}};
#pragma unroll
          for (int k = 0; k < 8; ++k) qs[k] = vad4(cf, quarter_win(hp, k, mixed, kh), qs[k]);
          ow = on;
          oc = ocn;
        }
      }
      ring_update<RD>(qs, xm, 1, bvx, bvy, P.lambda, qpx, qpy, best, bvx, bvy);
    }
    if (writer && (bx & xm) == 0) {
      P.out_qmvs[o + p] = (uint32_t)(uint16_t)bvx | ((uint32_t)(uint16_t)bvy << 16);
      const uint32_t d = best - (RD ? P.lambda * (se_bits(bvx - qpx) + se_bits(bvy - qpy)) : 0);
      P.out_sads[o + p] = (uint16_t)min(d, 65535u);
    }
  }
}

// CTA = one group of 8 MBs (gi) of MB row mrow of RF ref, 7 warps = the 7 modes.
template <bool RD>
__global__ void __launch_bounds__(kSme2Threads, FEVES_SME2_MINB) sme_smem_kernel(const SmeParams P, int* ovf) {
  extern __shared__ __align__(16) uint8_t sm2[];
  const int gid = blockIdx.x;                               // = the global kernel's warp index
  const int groups = (P.mb_cols + kSme2Mb - 1) / kSme2Mb;
  const int gi = gid % groups, rem = gid / groups;
  const int mrow = rem % P.n_rows, ref = rem / P.n_rows;
  const int mby = P.row0 + mrow;
  const int nmb = min(kSme2Mb, P.mb_cols - kSme2Mb * gi);   // MBs in this group
  const uint8_t* __restrict__ sf = P.sf[ref];
  const uint32_t s0 = (uint32_t)__cvta_generic_to_shared(sm2);
  const uint32_t s_cf = s0, s_mv = s0 + kSme2Mb * 256, s_sad = s_mv + kSme2Mb * 41 * 4;
  const uint32_t s_box = s_sad + kSme2Mb * 41 * 2;
  static_assert((kSme2Mb * (256 + 41 * 4 + 41 * 2)) % 8 == 0, "mbarrier alignment");
  const uint32_t s_reg = s0 + kSme2Head;
  const int tid = threadIdx.x;
  int* box4 = reinterpret_cast<int*>(sm2 + (s_box - s0));   // min x, max x, min y, max y
  const uint32_t bar = s_box + 16;                           // mbarrier of the staging copies
  if (tid < 4) box4[tid] = (tid & 1) ? -(1 << 30) : (1 << 30);
  if (tid == 0) mbar_init(bar, 1);
  __syncthreads();

  // ---- the group's ME results and the bounding box of their sub-pel footprints ----
  int xlo = 1 << 30, xhi = -(1 << 30), ylo = 1 << 30, yhi = -(1 << 30);
  for (int i = tid; i < kSme2Mb * kNPart; i += kSme2Threads) {
    const int g = i / kNPart, p = i - g * kNPart;
    const int mbx = kSme2Mb * gi + min(g, nmb - 1);
    const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
    const uint32_t mv = __ldg(P.in_mvs + o);
    const uint16_t sd = __ldg(P.in_sads + o);
    sts32(s_mv + 4 * i, mv);
    asm volatile("st.shared.u16 [%0], %1;" ::"r"(s_sad + 2 * i), "h"(sd));
    const int x = 16 * mbx + part_ox(p) + (int)(int16_t)(mv & 0xffffu);
    const int y = 16 * mby + part_oy(p) + (int)(int16_t)(mv >> 16);
    xlo = min(xlo, x - 1); xhi = max(xhi, x + part_w(p) + 1);
    ylo = min(ylo, y - 1); yhi = max(yhi, y + part_h(p) + 1);
  }
  xlo = __reduce_min_sync(0xffffffffu, xlo); xhi = __reduce_max_sync(0xffffffffu, xhi);
  ylo = __reduce_min_sync(0xffffffffu, ylo); yhi = __reduce_max_sync(0xffffffffu, yhi);
  if ((tid & 31) == 0) {
    atomicMin(box4 + 0, xlo); atomicMax(box4 + 1, xhi); atomicMin(box4 + 2, ylo); atomicMax(box4 + 3, yhi);
  }
  __syncthreads();
  xlo = box4[0]; xhi = box4[1]; ylo = box4[2]; yhi = box4[3];
  const int X0 = (xlo + P.pad) & ~15, X1 = (xhi + P.pad + 15) & ~15;   // plane columns, 16-byte aligned
  const int CW = X1 - X0, RH = yhi - ylo;                    // copied bytes per row
  const int WB = (CW + FEVES_SME2_PITCH - 1) & ~(FEVES_SME2_PITCH - 1);   // staged row pitch
  if (4 * WB * RH > FEVES_SME2_REGION) {                   // does not fit: global-load code afterwards
    if (tid == 0) {
      const int k = atomicAdd(ovf, 1);
      ovf[1 + k] = gid;
    }
    return;
  }
  // ---- stage 4 planes (G, b, h, j) x RH rows x WB bytes: one TMA bulk copy per row (one
  // thread each, completing on the mbarrier), and the CF rows through registers ----
  {
    if (tid == 0) mbar_expect_tx(bar, (uint32_t)(4 * CW * RH));
    int k = 0, rr = tid;                                   // row tid of the 4 * RH (plane, row) pairs
    while (rr >= RH && k < 4) { rr -= RH; ++k; }
    for (; k < 4;) {
      const int ph = (k & 1) * 2 + (k >> 1) * 8;          // plane index: 0 G, 2 b, 8 h, 10 j
      bulk_g2s(s_reg + (uint32_t)((k * RH + rr) * WB),
               sf + (size_t)ph * P.plane + (size_t)(ylo + rr + P.pad) * P.pitch + X0, (uint32_t)CW, bar);
      rr += kSme2Threads;
      while (rr >= RH && k < 4) { rr -= RH; ++k; }
    }
    for (int i = tid; i < kSme2Mb * 64; i += kSme2Threads) {   // CF: MBs x 16 rows x 4 words
      const int g = i >> 6, r = (i >> 2) & 15, q = i & 3;
      const int mbx = kSme2Mb * gi + min(g, nmb - 1);
      sts32(s_cf + 4 * i, load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * q, 16 * mby + r));
    }
    __syncthreads();
    mbar_wait(bar, 0);
  }
  const Box B{s_reg, (uint32_t)(WB * RH), (uint32_t)WB, ylo, P.pad - X0};

  // ---- lane group = mode, lane = (MB g, strip bx) ----
  const int m = sme2_mode(tid), g = (tid % kSme2Lpm) >> 2, bx = tid & 3;
  const bool writer = g < nmb && m < 7;
  const int gg = min(g, nmb - 1);
  const int mbx = kSme2Mb * gi + gg;
  const int xs = 16 * mbx + 4 * bx, ys0 = 16 * mby;
  const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart;
  int qpx = 0, qpy = 0;
  if (RD && P.pmv) {
    const size_t pi = ((size_t)mby * P.mb_cols + mbx) * P.rf_stride + ref;
    qpx = 4 * min(max((int)P.pmv[2 * pi], -P.max_pmv), P.max_pmv);
    qpy = 4 * min(max((int)P.pmv[2 * pi + 1], -P.max_pmv), P.max_pmv);
  }
  refine_mode_s<RD>(P, B, m == 7 ? 5 : m, s_cf, s_mv, s_sad, gg, bx, xs, ys0, writer, o, qpx, qpy);
  if (P.fence) __threadfence_system();
}

// Overflow groups of sme_smem_kernel (box larger than the region): the global-load
// refinement of sme_refine.cuh on the listed groups (warp = group x mode, as sme_refine_kernel),
// a small grid striding over the list (its length is known on the device only).
template <bool RD>
__global__ void __launch_bounds__(128, FEVES_SME_MINB) sme_list_kernel(const SmeParams P, const int* ovf) {
  const int count = *ovf;
  constexpr int kPer = 32 / kSme2Lpm;                        // listed groups per warp
  const int lane = threadIdx.x & 31, bx = lane & 3;
  const int groups = (P.mb_cols + kSme2Mb - 1) / kSme2Mb;
  const int n_w = (count + kPer - 1) / kPer;
  for (int w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < n_w; w += gridDim.x * (blockDim.x >> 5)) {
    const int li = kPer * w + lane / kSme2Lpm;
    const int warp_id = ovf[1 + min(li, count - 1)];
    const int gi = warp_id % groups, rem = warp_id / groups;
    const int mrow = rem % P.n_rows, ref = rem / P.n_rows;
    const int mbx_raw = kSme2Mb * gi + ((lane % kSme2Lpm) >> 2);
    const bool writer = li < count && mbx_raw < P.mb_cols;
    const int mbx = min(mbx_raw, P.mb_cols - 1);
    const int mby = P.row0 + mrow;
    const int xs = 16 * mbx + 4 * bx, ys0 = 16 * mby;
    const uint8_t* __restrict__ sf = P.sf[ref];
    const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart;
    int qpx = 0, qpy = 0;
    if (RD && P.pmv) {
      const size_t pi = ((size_t)mby * P.mb_cols + mbx) * P.rf_stride + ref;
      qpx = 4 * min(max((int)P.pmv[2 * pi], -P.max_pmv), P.max_pmv);
      qpy = 4 * min(max((int)P.pmv[2 * pi + 1], -P.max_pmv), P.max_pmv);
    }
    switch (blockIdx.y) {
      case 0: refine_mode<0, 4, 3, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      case 1: refine_mode<1, 2, 3, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      case 2: refine_mode<2, 4, 1, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      case 3: refine_mode<3, 2, 1, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      case 4: refine_mode<4, 1, 1, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      case 5: refine_mode<5, 2, 0, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
      default: refine_mode<6, 1, 0, RD, false>(P, sf, o, bx, xs, ys0, writer, qpx, qpy); break;
    }
  }
  if (P.fence) __threadfence_system();
}

}  // namespace feves
