// me_fsbm_pf.cuh -- the integer FSBM ME kernel (me_fsbm.cuh) as a PERSISTENT kernel whose
// search-area window loads are prefetched one window ahead ("TMA/shared-memory
// staging of the SA window plus halo per MB tile"; a2-a4 unchanged).
//
// me_fsbm_kernel stages every (MB, RF) window synchronously between two barriers: its global
// loads are exposed latency, and with one-warp CTAs (S = 32) or few candidates per window
// (S = 16) that latency is a large share of the kernel (ncu at 1080p S32: long_scoreboard
// 14.6%, ALU pipe 72.8% vs 80% at S = 64).  Here a CTA walks (MB, RF) windows w = k * grid +
// blockIdx.x (MB-major): while window w is searched, the raw rows of window w+1 (copy 0 of
// the 4 byte-shifted copies) and, at an MB change, the next CF rows are already in flight as
// 16-byte cp.async into a second buffer; at the next window the 3 shifted copies are built
// from shared memory (LDS + PRMT + STS, no global latency).  The candidate sweep, key-sum
// aggregation and (SAD, spiral rank) argmin are the same code as me_fsbm_kernel; results
// are identical (tested against the oracle).  Pure SAD, S = 16 / 32 / 64 (key-sum).
#pragma once
#include "me_fsbm.cuh"

namespace feves {

__host__ __device__ constexpr int me_pf_smem_words(int S) {
  return 2 * 64 + 5 * me_cstride(S) + (me_threads(S) / 32) * kNPart;   // 2 CF, 5 window slots, reduction
}

__device__ __forceinline__ void pf_cp16(uint32_t* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(src));
}

template <int S_CT>
__global__ void __launch_bounds__(128, FEVES_ME_MINB) me_pf_kernel(const MeParams P, int n_items) {
  static_assert(S_CT == 16 || S_CT == 32 || S_CT == 64, "key-sum sizes");
  extern __shared__ __align__(16) uint32_t smem[];
  constexpr int S = S_CT, R = S / 2, hi = S - 1 - R;
  constexpr int PW = me_pw(S), CSTRIDE = me_cstride(S), LX = me_lx(S), NGX = me_ngx(S);
  constexpr int NSUB = me_nsub(S), DYL = me_dyl(S);
  constexpr int WROWS = S + 15, CHUNKS = PW / 4;
  uint32_t* cf_buf = smem;                                // [2][64]: CF rows of the current / next MB
  uint32_t* win = smem + 128;                             // slots 0..4: c0 (even windows), c1, c2, c3, c0 (odd)
  uint32_t* red = win + 5 * CSTRIDE;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  const uint32_t one = (uint32_t)(P.n_rf > 0);            // == 1, opaque to the compiler (see fadd)
  const int gx = warp % NGX, wy = me_nwy(S) > 1 ? warp / NGX : 0;
  const int xi = lane % LX, sub = wy * NSUB + lane / LX;
  const int dx = min(-R + gx * LX + xi, hi);
  const int off = dx + R;
  const int dy_begin = -R + sub * DYL;
  const uint32_t* rank_col = P.rank_tab + off * me_rank_pitch(S) + R;
  const int n_win = n_items * P.n_rf;

  // issue the loads of window w (raw rows -> c0 slot `slot`) and, for its first RF, the MB's CF
  // rows (-> CF buffer `cslot`); both buffers alternate per window / per MB of THIS CTA
  auto prefetch = [&](int w, int slot, int cslot) {
    const int item = w / P.n_rf, ref = w - item * P.n_rf;
    const int mbx = item % P.mb_cols, mby = P.row0 + item / P.mb_cols;
    const uint8_t* __restrict__ rf = P.rf[ref];
    uint32_t* c0 = win + (slot ? 4 : 0) * CSTRIDE;
    const int xw0 = 16 * mbx - R, yw0 = 16 * mby - R;
    for (int it = threadIdx.x; it < WROWS * CHUNKS; it += blockDim.x) {
      const int row = it / CHUNKS, k = it - row * CHUNKS;
      const int x = xw0 + 16 * k, y = min(max(yw0 + row, 0), P.H - 1);
      uint32_t* dst = c0 + row * PW + 4 * k;
      if (P.vec_ok && x >= 0 && x + 16 <= P.W) {
        pf_cp16(dst, rf + (size_t)y * P.W + x);
      } else {
        *reinterpret_cast<uint4*>(dst) = make_uint4(load4_clamped(rf, P.W, P.H, x, y), load4_clamped(rf, P.W, P.H, x + 4, y),
                                                    load4_clamped(rf, P.W, P.H, x + 8, y), load4_clamped(rf, P.W, P.H, x + 12, y));
      }
    }
    if (ref == 0) {
      uint32_t* cf_s = cf_buf + 64 * cslot;
      for (int i = threadIdx.x; i < 16; i += blockDim.x) {   // one 16-byte CF row per thread
        const int x = 16 * mbx, y = 16 * mby + i;
        if (P.cf_vec16 && x + 16 <= P.W && y < P.H) {
          pf_cp16(cf_s + 4 * i, P.cf + (size_t)y * P.W + x);
        } else {
          *reinterpret_cast<uint4*>(cf_s + 4 * i) =
              make_uint4(load4_clamped(P.cf, P.W, P.H, x, y), load4_clamped(P.cf, P.W, P.H, x + 4, y),
                         load4_clamped(P.cf, P.W, P.H, x + 8, y), load4_clamped(P.cf, P.W, P.H, x + 12, y));
        }
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };

  int w = blockIdx.x * P.n_rf;                            // the CTA's windows: item-major
  int kw = 0, ki = 0;                                     // windows / MBs this CTA has started
  if (w < n_win) prefetch(w, 0, 0);
  for (; w < n_win; ++kw) {
    const int item = w / P.n_rf, ref = w - item * P.n_rf;
    const int mbx = item % P.mb_cols, mrow = item / P.mb_cols;
    uint32_t* c0 = win + ((kw & 1) ? 4 : 0) * CSTRIDE;
    const uint32_t* cf_s = cf_buf + 64 * (ki & 1);
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncthreads();                                      // raw window + CF visible; the previous window is done
    // ---- the 3 byte-shifted copies from the raw rows (copy c word q = raw bytes [4q+c, 4q+c+4)) ----
    for (int it = threadIdx.x; it < WROWS * CHUNKS; it += blockDim.x) {
      const int row = it / CHUNKS, k = it - row * CHUNKS;
      const uint32_t* src = c0 + row * PW + 4 * k;
      const uint4 a = *reinterpret_cast<const uint4*>(src);
      const uint32_t n = (k + 1 < CHUNKS) ? src[4] : 0u;  // the last word of a row is never read shifted
      uint32_t* dst = win + row * PW + 4 * k;
      *reinterpret_cast<uint4*>(dst + CSTRIDE) = make_uint4(__byte_perm(a.x, a.y, 0x4321), __byte_perm(a.y, a.z, 0x4321),
                                                            __byte_perm(a.z, a.w, 0x4321), __byte_perm(a.w, n, 0x4321));
      *reinterpret_cast<uint4*>(dst + 2 * CSTRIDE) = make_uint4(__byte_perm(a.x, a.y, 0x5432), __byte_perm(a.y, a.z, 0x5432),
                                                                __byte_perm(a.z, a.w, 0x5432), __byte_perm(a.w, n, 0x5432));
      *reinterpret_cast<uint4*>(dst + 3 * CSTRIDE) = make_uint4(__byte_perm(a.x, a.y, 0x6543), __byte_perm(a.y, a.z, 0x6543),
                                                                __byte_perm(a.z, a.w, 0x6543), __byte_perm(a.w, n, 0x6543));
    }
    __syncthreads();
    const bool last_ref = ref + 1 == P.n_rf;
    const int wn = last_ref ? w - ref + gridDim.x * P.n_rf : w + 1;
    if (wn < n_win) prefetch(wn, (kw + 1) & 1, (ki + (last_ref ? 1 : 0)) & 1);   // in flight during this sweep

    // ---- a2-a4: the candidate sweep of me_fsbm_kernel (key-sum aggregation) ----
    const uint32_t* wbase = ((off & 3) ? win + (off & 3) * CSTRIDE : c0) + (off >> 2);
    uint32_t M[kNPart];
#pragma unroll
    for (int p = 0; p < kNPart; ++p) M[p] = 0xffffffffu;
    uint32_t rank_next[kMeT];
    auto load_ranks = [&](int d0) {
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(rank_col + d0));
      rank_next[0] = v.x; rank_next[1] = v.y; rank_next[2] = v.z; rank_next[3] = v.w;
    };
    load_ranks(min(dy_begin, hi + 1 - kMeT));
    for (int c = 0; c < DYL; c += kMeT) {
      const int dy0 = min(dy_begin + c, hi + 1 - kMeT);
      uint32_t rank[kMeT];
#pragma unroll
      for (int t = 0; t < kMeT; ++t) rank[t] = rank_next[t];
      load_ranks(min(dy_begin + c + kMeT, hi + 1 - kMeT));
      const uint32_t* wrow = wbase + (dy0 + R) * PW;
      uint32_t acc[kMeT][4];
      RowState st[kMeT];
      uint32_t Kp[kMeT][16];
      uint4 cfr[16];
#pragma unroll
      for (int i = 0; i < kMeT + 15; ++i) {
        if (i < 16) cfr[i] = lds128_v(cf_s + 4 * i);
        uint32_t wv[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) wv[b] = wrow[i * PW + b];
#pragma unroll
        for (int b = 0; b < 4; ++b)
#pragma unroll
          for (int t = 0; t < kMeT; ++t) {
            const int r = i - t;
            if (r >= 0 && r < 16) {
              const uint32_t cw[4] = {cfr[r].x, cfr[r].y, cfr[r].z, cfr[r].w};
              acc[t][b] = vad4(cw[b], wv[b], (r & 3) ? acc[t][b] : 0u);
            }
          }
#pragma unroll
        for (int t = 0; t < kMeT; ++t) {
          const int r = i - t;
          if (r >= 0 && r < 16 && (r & 3) == 3) {
            const int by = r >> 2;
            if (by == 0) block_row_keys_sum<0>(acc[t], rank[t], st[t], Kp[t], one);
            if (by == 1) block_row_keys_sum<1>(acc[t], rank[t], st[t], Kp[t], one);
            if (by == 2) block_row_keys_sum<2>(acc[t], rank[t], st[t], Kp[t], one);
            if (by == 3) block_row_keys_sum<3>(acc[t], rank[t], st[t], Kp[t], one);
            if (t & 1) {
              if (by == 0) fold_pair<0>(M, Kp[t - 1], Kp[t]);
              if (by == 1) fold_pair<1>(M, Kp[t - 1], Kp[t]);
              if (by == 2) fold_pair<2>(M, Kp[t - 1], Kp[t]);
              if (by == 3) fold_pair<3>(M, Kp[t - 1], Kp[t]);
            }
          }
        }
      }
    }
    // ---- warp min (CREDUX), CTA min, rank -> MV ----
#pragma unroll
    for (int p = 0; p < kNPart; ++p) {
      const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
      if (lane == 0) red[warp * kNPart + p] = v;
    }
    __syncthreads();
    for (int p = threadIdx.x; p < kNPart; p += blockDim.x) {
      uint32_t k = red[p];
      for (int ww = 1; ww < nwarps; ++ww) k = min(k, red[ww * kNPart + p]);
      const uint32_t rk = (k & 0xffffu) >> part_log2n(p);
      const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
      reinterpret_cast<uint32_t*>(P.out_mvs)[o] = __ldg(P.inv_tab + rk);
      P.out_sads[o] = (uint16_t)(k >> 16);
    }
    w = wn;
    ki += last_ref ? 1 : 0;
  }
}

}  // namespace feves
