// me_fsbm_rfp.cuh -- integer FSBM ME, RF-parallel CTA (S = 64, pure SAD).
// EXPERIMENT (not built into libfeves_me.so): measured slower than me_fsbm_kernel, see DESIGN.md §6.
//
// Same computation, lane geometry, key-sum aggregation and argmin as me_fsbm_kernel<64>
// (me_fsbm.cuh; P:6, readings G1-G7): what changes is how a CTA walks the RFs.  One CTA =
// one MB and up to RFP = 4 of its RFs AT ONCE: warp pair f (2 warps = the 64 dx of the SA)
// searches RF rg + f, so the 4 SA windows are staged in ONE phase (all their global loads
// in flight together, one barrier) instead of 4 stage -> barrier -> search rounds, and the
// warp/CTA reduction runs once per RF group.  Shared memory: 4 windows x 25.7 KB -> 2 CTAs
// (16 warps) per SM, the same occupancy as 8 CTAs of 2 warps.
#pragma once
#include "../../paper_conf_icpp_ilicmrs14_b200/csrc/me_fsbm.cuh"

namespace feves {

constexpr int kRfp = 4;   // RFs searched concurrently by one CTA
__host__ __device__ constexpr int rfp_threads(int rfp) { return 64 * rfp; }
__host__ __device__ constexpr int rfp_smem_words(int rfp) { return 64 + rfp * 4 * me_cstride(64) + 2 * rfp * kNPart; }

__global__ void __launch_bounds__(64 * kRfp, 2) me_fsbm_rfp_kernel(const MeParams P) {
  extern __shared__ __align__(16) uint32_t smem[];
  constexpr int S = 64, R = 32, hi = S - 1 - R;
  constexpr int PW = me_pw(S), CSTRIDE = me_cstride(S), win_rows = S + 15, chunks = PW >> 2;
  const int rfp = blockDim.x >> 6;                        // RFs per group (<= kRfp)
  uint32_t* cf_s = smem;                                  // 16 rows x 4 words
  uint32_t* win_all = smem + 64;                          // rfp windows x 4 copies x CSTRIDE words
  uint32_t* red = win_all + rfp * 4 * CSTRIDE;            // [2 * rfp warps][41]

  const int mbx = blockIdx.x, mby = P.row0 + blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int f = warp >> 1;                                // RF slot of this warp pair
  const uint32_t one = (uint32_t)(P.n_rf > 0);
  const int dx = -R + 32 * (warp & 1) + lane;
  const int off = dx + R;
  const uint32_t* wbase = win_all + f * 4 * CSTRIDE + (off & 3) * CSTRIDE + (off >> 2);
  const uint32_t* rank_col = P.rank_tab + off * me_rank_pitch(S) + R;

  for (int i = threadIdx.x; i < 64; i += blockDim.x)
    cf_s[i] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * (i & 3), 16 * mby + (i >> 2));
  const int xw0 = 16 * mbx - R, yw0 = 16 * mby - R;

  for (int rg = 0; rg < P.n_rf; rg += rfp) {
    const int nf = min(rfp, P.n_rf - rg);                 // RFs in this group
    __syncthreads();
    // ---- a1: the nf windows, 4 byte-shifted copies each (as me_fsbm_kernel) ----
    for (int item = threadIdx.x; item < nf * win_rows * chunks; item += blockDim.x) {
      const int fi = item / (win_rows * chunks), r2 = item - fi * win_rows * chunks;
      const int row = r2 / chunks, k = r2 - row * chunks;
      const uint8_t* __restrict__ rf = P.rf[rg + fi];
      const int x = xw0 + 16 * k, y = min(max(yw0 + row, 0), P.H - 1);
      uint32_t w[5];
      if (P.vec_ok && x >= 0 && x + 20 <= P.W) {
        const uint8_t* src = rf + (size_t)y * P.W + x;
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(src));
        w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
        w[4] = __ldg(reinterpret_cast<const uint32_t*>(src + 16));
      } else {
#pragma unroll
        for (int i = 0; i < 5; ++i) w[i] = load4_clamped(rf, P.W, P.H, x + 4 * i, y);
      }
      uint32_t* dst = win_all + fi * 4 * CSTRIDE + row * PW + 4 * k;
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
    __syncthreads();

    if (f < nf) {                                         // warp-uniform
      uint32_t M[kNPart];
#pragma unroll
      for (int p = 0; p < kNPart; ++p) M[p] = 0xffffffffu;
      uint4 rank_next = __ldg(reinterpret_cast<const uint4*>(rank_col - R));
      for (int c = 0; c < S; c += kMeT) {
        const int dy0 = -R + c;
        const uint32_t rank[4] = {rank_next.x, rank_next.y, rank_next.z, rank_next.w};
        rank_next = __ldg(reinterpret_cast<const uint4*>(rank_col + min(dy0 + kMeT, hi + 1 - kMeT)));
        const uint32_t* wrow = wbase + (dy0 + R) * PW;
        uint32_t acc[kMeT][4];
        RowState st[kMeT];
        uint32_t Kp[kMeT][16];
        uint4 cfr[16];
#pragma unroll
        for (int i = 0; i < kMeT + 15; ++i) {
          if (i < 16) cfr[i] = lds128_v(cf_s + 4 * i);
          uint32_t w[4];
#pragma unroll
          for (int b = 0; b < 4; ++b) w[b] = wrow[i * PW + b];
#pragma unroll
          for (int t = 0; t < kMeT; ++t) {
            const int r = i - t;
            if (r >= 0 && r < 16) {
              const uint32_t cw[4] = {cfr[r].x, cfr[r].y, cfr[r].z, cfr[r].w};
#pragma unroll
              for (int b = 0; b < 4; ++b) acc[t][b] = vad4(cw[b], w[b], (r & 3) ? acc[t][b] : 0u);
              if ((r & 3) == 3) {
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
      }
#pragma unroll
      for (int p = 0; p < kNPart; ++p) {
        const uint32_t v = __reduce_min_sync(0xffffffffu, M[p]);
        if (lane == 0) red[warp * kNPart + p] = v;
      }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < nf * kNPart; i += blockDim.x) {
      const int fi = i / kNPart, p = i - fi * kNPart;
      const uint32_t k = min(red[(2 * fi) * kNPart + p], red[(2 * fi + 1) * kNPart + p]);
      const uint32_t mv = __ldg(P.inv_tab + ((k & 0xffffu) >> part_log2n(p)));
      const size_t o = ((size_t)(blockIdx.y * P.mb_cols + mbx) * P.rf_stride + rg + fi) * kNPart + p;
      reinterpret_cast<uint32_t*>(P.out_mvs)[o] = mv;
      P.out_sads[o] = (uint16_t)(k >> 16);
    }
  }
}

}  // namespace feves
