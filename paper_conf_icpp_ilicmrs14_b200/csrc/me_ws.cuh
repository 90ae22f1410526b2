// me_ws.cuh -- warp-specialised integer FSBM ME for sm_100a, S = 64.
//
// Same arithmetic as me_fsbm_kernel (P:6: SAD over the SA of every MB in every RF, 41
// partitions, minimum distortion; key = SAD * 2^16 + dense spiral rank, key-sum
// aggregation, VIMNMX3 folds, G4 tie-break) -- only the work split inside the CTA differs.
//
// Why: in me_fsbm_kernel every warp stages its RF window (dependent global loads + a
// barrier) and reduces its minima (CREDUX, barrier, a dependent rank-table load) between
// two candidate sweeps; ncu samples ~24% of the warp time outside the candidate loop, and
// the loop's ALU pipe reaches 81% where the same instruction mix alone reaches 86-89% at
// 2-3 warps per scheduler (profiles/r02/mix_pipes_ncu.txt).  Here the CTA is
//   warp 0      producer: stages the (S+15)^2 window of RF r+1 (4 byte-shifted copies, as
//               me_fsbm_kernel) into the other half of a double buffer while the
//               compute warps sweep RF r, then reduces RF r's warp minima to the CTA
//               minimum and writes the MVs / SADs;
//   warps 1-4   compute: (dx group, dy half) of the 64 x 64 candidates, 8 chunks of
//               T = 4 dy per RF, the same candidate loop; they only wait on a barrier
//               when the next window is not staged yet.
// Hand-offs are named barriers (bar.arrive / bar.sync, 160 threads):
//   FULL(b)  producer arrives after staging buffer b, compute warps sync on it;
//   DONE(b)  compute warps arrive after their sweep of buffer b and after storing their
//            warp minima into red[b]; the producer syncs on it before the epilogue of
//            that RF (and therefore before restaging b two RFs later).
// Shared memory: 2 x CF 64 words + 2 windows x 4 copies x CSTRIDE + 2 x 4 x 41 minima (53 KB:
// 3 CTAs = 12 compute warps per SM, registers capped at 136 by the launch bounds).
#pragma once
#include "me_fsbm.cuh"

namespace feves {

constexpr int kWsS = 64;
#ifndef FEVES_WS_CW
#define FEVES_WS_CW 4
#endif
constexpr int kWsCw = FEVES_WS_CW;                        // compute warps: 2 dx groups x (kWsCw / 2) dy slices
constexpr int kWsThreads = 32 * (1 + kWsCw);
constexpr int kWsDyl = kWsS / (kWsCw / 2);                // dy per compute warp (chunks of 4)
constexpr int kWsMinB = kWsCw == 4 ? 3 : 4;               // resident CTAs per SM (53 KB of shared memory each)
__host__ __device__ constexpr int me_ws_smem_words() { return 128 + 2 * 4 * me_cstride(kWsS) + 2 * kWsCw * kNPart; }

// named barriers with compile-time ids (ptxas then reserves only ids 0..4): FULL(b) = 1 + b,
// DONE(b) = 3 + b; b = buffer parity (run time, warp-uniform)
template <int ID>
__device__ __forceinline__ void ws_sync_id() { asm volatile("bar.sync %0, %1;" ::"n"(ID), "n"(kWsThreads) : "memory"); }
template <int ID>
__device__ __forceinline__ void ws_arrive_id() { asm volatile("bar.arrive %0, %1;" ::"n"(ID), "n"(kWsThreads) : "memory"); }
__device__ __forceinline__ void ws_full_arrive(int b) { if (b) ws_arrive_id<2>(); else ws_arrive_id<1>(); }
__device__ __forceinline__ void ws_full_sync(int b) { if (b) ws_sync_id<2>(); else ws_sync_id<1>(); }
__device__ __forceinline__ void ws_done_arrive(int b) { if (b) ws_arrive_id<4>(); else ws_arrive_id<3>(); }
__device__ __forceinline__ void ws_done_sync(int b) { if (b) ws_sync_id<4>(); else ws_sync_id<3>(); }

#ifndef FEVES_WS_NB
#define FEVES_WS_NB 13  // window items per lane whose loads the producer issues back to back (13 x 32 >= 395: one round trip)
#endif

// producer: stage the SA window of RF `rf` (rows yst .. yst + S + 14, columns xw0 .. +PW*4)
// into the 4 byte-shifted copies at win (same layout as me_fsbm_kernel's a1)
__device__ __forceinline__ void ws_stage(const MeParams& P, const uint8_t* __restrict__ rf, uint32_t* win, int xw0,
                                         int yst, int lane) {
  constexpr int PW = me_pw(kWsS), CSTRIDE = me_cstride(kWsS), ROWS = kWsS + 15, CHUNKS = PW >> 2;
  constexpr int ITEMS = ROWS * CHUNKS;
#pragma unroll 1
  for (int base = 0; base < ITEMS; base += 32 * FEVES_WS_NB) {
    uint32_t w[FEVES_WS_NB][5];
#pragma unroll
    for (int j = 0; j < FEVES_WS_NB; ++j) {              // all loads first: NB round trips overlap
      const int item = base + 32 * j + lane;
      if (item < ITEMS) {
        const int row = item / CHUNKS, k = item - row * CHUNKS;
        const int x = xw0 + 16 * k, y = min(max(yst + row, 0), P.H - 1);
        if (P.vec_ok && x >= 0 && x + 20 <= P.W) {
          const uint8_t* src = rf + (size_t)y * P.W + x;
          const uint4 v = __ldg(reinterpret_cast<const uint4*>(src));
          w[j][0] = v.x; w[j][1] = v.y; w[j][2] = v.z; w[j][3] = v.w;
          w[j][4] = __ldg(reinterpret_cast<const uint32_t*>(src + 16));
        } else {
#pragma unroll
          for (int i = 0; i < 5; ++i) w[j][i] = load4_clamped(rf, P.W, P.H, x + 4 * i, y);
        }
      }
    }
#pragma unroll
    for (int j = 0; j < FEVES_WS_NB; ++j) {
      const int item = base + 32 * j + lane;
      if (item < ITEMS) {
        const int row = item / CHUNKS, k = item - row * CHUNKS;
        uint32_t* dst = win + row * PW + 4 * k;
        *reinterpret_cast<uint4*>(dst) = make_uint4(w[j][0], w[j][1], w[j][2], w[j][3]);
        *reinterpret_cast<uint4*>(dst + CSTRIDE) =
            make_uint4(__byte_perm(w[j][0], w[j][1], 0x4321), __byte_perm(w[j][1], w[j][2], 0x4321),
                       __byte_perm(w[j][2], w[j][3], 0x4321), __byte_perm(w[j][3], w[j][4], 0x4321));
        *reinterpret_cast<uint4*>(dst + 2 * CSTRIDE) =
            make_uint4(__byte_perm(w[j][0], w[j][1], 0x5432), __byte_perm(w[j][1], w[j][2], 0x5432),
                       __byte_perm(w[j][2], w[j][3], 0x5432), __byte_perm(w[j][3], w[j][4], 0x5432));
        *reinterpret_cast<uint4*>(dst + 3 * CSTRIDE) =
            make_uint4(__byte_perm(w[j][0], w[j][1], 0x6543), __byte_perm(w[j][1], w[j][2], 0x6543),
                       __byte_perm(w[j][2], w[j][3], 0x6543), __byte_perm(w[j][3], w[j][4], 0x6543));
      }
    }
  }
}

// Persistent CTAs: CTA c takes the MBs c, c + gridDim.x, ... of the stripe (static order, so
// producer and compute warps walk the same job sequence without talking); a job = (MB, RF),
// job j uses window buffer j & 1, MB i of the CTA uses CF buffer i & 1.  The producer stages
// job j + 1 (and the CF of the next MB) during job j's sweep, so a CTA pays one exposed
// staging at its start, not one per MB.
__global__ void __launch_bounds__(kWsThreads, kWsMinB) me_ws_kernel(const MeParams P, int n_mb) {
  extern __shared__ __align__(16) uint32_t smem[];
  constexpr int S = kWsS, R = S / 2, PW = me_pw(S), CSTRIDE = me_cstride(S);
  uint32_t* cfs = smem;                                   // [2][16 rows x 4 words]
  uint32_t* wins = smem + 128;                            // [2][4 copies][CSTRIDE]
  uint32_t* red = wins + 2 * 4 * CSTRIDE;                 // [2][kWsCw][41]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = gridDim.x;
  if (P.n_rf <= 0 || (int)blockIdx.x >= n_mb) return;
  const int my_mbs = (n_mb - 1 - (int)blockIdx.x) / G + 1;
  const int n_jobs = my_mbs * P.n_rf;
  auto mb_of = [&](int i, int& mbx, int& mrow) {          // i-th MB of this CTA -> (column, stripe row)
    const int m = (int)blockIdx.x + i * G;
    mrow = m / P.mb_cols;
    mbx = m - mrow * P.mb_cols;
  };

  if (warp == 0) {
    // ------------------------------------------------------------ producer --
    auto stage_job = [&](int j) {                         // CF (first RF of an MB) + window of job j
      const int i = j / P.n_rf, ref = j - i * P.n_rf;
      int mbx, mrow;
      mb_of(i, mbx, mrow);
      const int mby = P.row0 + mrow;
      if (ref == 0) {
        uint32_t* cf_s = cfs + 64 * (i & 1);
        for (int q = lane; q < 64; q += 32)
          cf_s[q] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * (q & 3), 16 * mby + (q >> 2));
      }
      ws_stage(P, P.rf[ref], wins + (j & 1) * 4 * CSTRIDE, 16 * mbx - R, 16 * mby - R, lane);
      ws_full_arrive(j & 1);
    };
    stage_job(0);
    for (int j = 0; j < n_jobs; ++j) {
      if (j + 1 < n_jobs) stage_job(j + 1);               // buffer (j+1)&1 was released in epilogue(j-1)
      const int b = j & 1;
      ws_done_sync(b);                                    // the compute warps' minima of job j
      const int i = j / P.n_rf, ref = j - i * P.n_rf;
      int mbx, mrow;
      mb_of(i, mbx, mrow);
      const uint32_t* rb = red + b * kWsCw * kNPart;
      for (int p = lane; p < kNPart; p += 32) {           // a4: CTA minimum, rank -> (dx, dy)
        uint32_t k = rb[p];
#pragma unroll
        for (int w = 1; w < kWsCw; ++w) k = min(k, rb[w * kNPart + p]);
        const uint32_t rk = (k & 0xffffu) >> part_log2n(p);   // key-sum: n * rank in the low half
        const uint32_t mv = __ldg(P.inv_tab + rk);
        const size_t o = ((size_t)(mrow * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
        reinterpret_cast<uint32_t*>(P.out_mvs)[o] = mv;
        P.out_sads[o] = (uint16_t)(k >> 16);
      }
    }
    return;
  }

  // ------------------------------------------------------------- compute --
  const int cw = warp - 1;
  const int gx = cw & 1, wy = cw >> 1;
  const int dx = -R + gx * 32 + lane;                     // every lane a distinct dx (S = 64 = 2 x 32)
  const int off = dx + R;
  const int dy_begin = -R + wy * kWsDyl;
  const uint32_t one = (uint32_t)(P.n_rf > 0);            // == 1, opaque to the compiler (see fadd)
  const uint32_t* rank_col = P.rank_tab + off * me_rank_pitch(S) + R;

#pragma unroll 1
  for (int j = 0; j < n_jobs; ++j) {
    const int b = j & 1;
    const uint32_t* cf_s = cfs + 64 * ((j / P.n_rf) & 1);
    const uint32_t* wbase = wins + b * 4 * CSTRIDE + (off & 3) * CSTRIDE + (off >> 2);
    uint32_t M[kNPart];
#pragma unroll
    for (int p = 0; p < kNPart; ++p) M[p] = 0xffffffffu;
    uint32_t rank_next[kMeT];
    auto load_ranks = [&](int d0) {
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(rank_col + d0));
      rank_next[0] = v.x; rank_next[1] = v.y; rank_next[2] = v.z; rank_next[3] = v.w;
    };
    load_ranks(dy_begin);
    ws_full_sync(b);                                      // window (and CF) of job j staged
#pragma unroll 1
    for (int c = 0; c < kWsDyl; c += kMeT) {
      const int dy0 = dy_begin + c;
      uint32_t rank[kMeT];
#pragma unroll
      for (int t = 0; t < kMeT; ++t) rank[t] = rank_next[t];
      load_ranks(min(dy0 + kMeT, dy_begin + kWsDyl - kMeT));   // prefetch the next chunk's ranks
      const uint32_t* wrow = wbase + (dy0 + R) * PW;

      uint32_t acc[kMeT][4];
      RowState st[kMeT];
      uint32_t Kp[kMeT][16];
      uint4 cfr[16];
#pragma unroll
      for (int i = 0; i < kMeT + 15; ++i) {
        if (i < 16) cfr[i] = lds128_v(cf_s + 4 * i);     // CF row i, used by RF rows i..i+3
        uint32_t w[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) w[q] = wrow[i * PW + q];
#pragma unroll
        for (int q = 0; q < 4; ++q)
#pragma unroll
          for (int t = 0; t < kMeT; ++t) {
            const int r = i - t;
            if (r >= 0 && r < 16) {
              const uint32_t cw4[4] = {cfr[r].x, cfr[r].y, cfr[r].z, cfr[r].w};
              acc[t][q] = vad4(cw4[q], w[q], (r & 3) ? acc[t][q] : 0u);
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
    // warp minima -> red[b]; then release buffer b and hand the minima to the producer
    uint32_t* rb = red + b * kWsCw * kNPart + cw * kNPart;
#pragma unroll
    for (int p = 0; p < kNPart; ++p) {
      const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
      if (lane == (p & 31)) rb[p] = v;
    }
    ws_done_arrive(b);
  }
}

}  // namespace feves
