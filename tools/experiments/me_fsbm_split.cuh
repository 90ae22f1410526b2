// me_fsbm_split.cuh -- integer FSBM ME, "half-MB lane pair" variant (S = 32, 64; pure SAD).
// EXPERIMENT (not built into libfeves_me.so): measured slower than me_fsbm_kernel, see DESIGN.md §6.
//
// Same computation as me_fsbm_kernel (P:6, readings G1-G7): every
// candidate (dx,dy) of the S x S SA, all 41 partitions, key = SAD * 2^16 + dense rank,
// argmin with the spiral-rank tie-break (G4).  What changes is the lane geometry:
//
//  * two ADJACENT lanes share one candidate column dx: lane h = 0 takes the left 8 pixel
//    columns of the MB, lane h = 1 the right 8.  Each lane reads 2 window words per RF
//    row and holds half of the per-candidate state (2 accumulators per candidate instead
//    of 4, 4 carried keys instead of 9, 2 CF words per row instead of 4, 22 running
//    minima instead of 41), which is what lets 6 warps per scheduler be resident instead
//    of 4 for an ALU-pipe-bound kernel;
//  * the 19 partitions inside a half (8 4x4, 4 8x4, 4 4x8, 2 8x8, 1 8x16) are the lane's
//    own; the 3 partitions spanning both halves (16x8 top/bottom, 16x16) are formed by
//    both lanes of the pair from their 8x8 keys exchanged with one SHFL.BFLY each
//    (key-sum aggregation: parent key = sum of child keys, me_fsbm.cuh SumKeys);
//  * the warp/CTA reduction runs separately over the even and the odd lanes (the same
//    running-min slot holds a left-half partition on even lanes, a right-half one on odd).
//
// Per MB-candidate (both lanes): 64 VABSDIFF4 + 22 VIMNMX3 (ALU), 44 IMAD (FMA), 19 LDS +
// 8 LDS.64 + 4 SHFL.  Window staging, rank table and output layout are those of
// me_fsbm_kernel.
#pragma once
#include "../../paper_conf_icpp_ilicmrs14_b200/csrc/me_fsbm.cuh"

namespace feves {

__host__ __device__ constexpr int mes_threads(int S) { return 2 * S; }
__host__ __device__ constexpr int mes_smem_words(int S) {
  return 64 + 4 * me_cstride(S) + (mes_threads(S) / 32) * kNPart;
}

// running-min slot s of lane half h -> partition index (G7)
__host__ __device__ constexpr int mes_part(int s, int h) {
  return s < 8 ? 25 + 4 * (2 * ((s >> 1) >> 1) + h) + 2 * ((s >> 1) & 1) + (s & 1)     // 4x4 (by = s>>1, i = s&1)
       : s < 12 ? 9 + 2 * (2 * ((s - 8) >> 1) + h) + ((s - 8) & 1)                       // 8x4 (by = s-8)
       : s < 16 ? 17 + 2 * (2 * ((s - 12) >> 1) + h) + ((s - 12) & 1)                    // 4x8 (by pair, i)
       : s < 18 ? 5 + 2 * (s - 16) + h                                                   // 8x8 (top / bottom)
       : s == 18 ? 3 + h                                                                 // 8x16
       : s < 21 ? 1 + (s - 19)                                                           // 16x8 top / bottom
       : 0;                                                                              // 16x16
}
constexpr int kMesSlots = 22;

struct HalfState {
  uint32_t k4prev[2];   // keys of the upper 4x4s of the current block-row pair (for 4x8)
  uint32_t k84top;      // key of the upper 8x4 (for 8x8)
  uint32_t k88top;      // key of the top 8x8 (for 8x16)
  uint32_t k168top;     // key of the top 16x8 (for 16x16)
};

// keys completed by block row BY of one candidate, in slot order (KS = 22 slots; the
// entries of slots not completed by this block row are left untouched)
template <int BY>
__device__ __forceinline__ void half_row_keys(const uint32_t (&L)[2], uint32_t rank, HalfState& st,
                                              uint32_t (&K)[kMesSlots], uint32_t one) {
  const uint32_t k0 = kmad<16>(L[0], rank), k1 = kmad<16>(L[1], rank);   // 4x4
  K[2 * BY] = k0;
  K[2 * BY + 1] = k1;
  const uint32_t k84 = fadd(k0, k1, one);                                 // 8x4
  K[8 + BY] = k84;
  if ((BY & 1) == 0) {
    st.k4prev[0] = k0; st.k4prev[1] = k1; st.k84top = k84;
  } else {
    K[12 + 2 * (BY >> 1)] = fadd(k0, st.k4prev[0], one);                  // 4x8
    K[13 + 2 * (BY >> 1)] = fadd(k1, st.k4prev[1], one);
    const uint32_t k88 = fadd(k84, st.k84top, one);                       // 8x8
    K[16 + (BY >> 1)] = k88;
    const uint32_t k88o = __shfl_xor_sync(0xffffffffu, k88, 1);           // the other half's 8x8
    const uint32_t k168 = fadd(k88, k88o, one);                           // 16x8 (same on both lanes)
    K[19 + (BY >> 1)] = k168;
    if (BY == 1) {
      st.k88top = k88; st.k168top = k168;
    } else {
      K[18] = fadd(st.k88top, k88, one);                                  // 8x16
      K[21] = fadd(st.k168top, k168, one);                                // 16x16
    }
  }
}

template <int BY>
__device__ __forceinline__ void half_fold_pair(uint32_t (&M)[kMesSlots], const uint32_t (&Ka)[kMesSlots],
                                               const uint32_t (&Kb)[kMesSlots]) {
  // slots completed by block row BY
#pragma unroll
  for (int s = 0; s < kMesSlots; ++s) {
    const bool done = (s < 8) ? (s >> 1) == BY
                    : (s < 12) ? s - 8 == BY
                    : (s < 16) ? ((BY & 1) && ((s - 12) >> 1) == (BY >> 1))
                    : (s < 18) ? ((BY & 1) && s - 16 == (BY >> 1))
                    : (s == 18) ? BY == 3
                    : (s < 21) ? ((BY & 1) && s - 19 == (BY >> 1))
                    : BY == 3;
    if (done) M[s] = umin3(M[s], Ka[s], Kb[s]);
  }
}

__device__ __forceinline__ uint2 lds64_v(const uint32_t* p) {
  uint2 v;
  const unsigned a = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}

#ifndef FEVES_MES_MINB
#define FEVES_MES_MINB 6
#endif
template <int S>
__global__ void __launch_bounds__(2 * S, (S == 64 ? FEVES_MES_MINB : 2 * FEVES_MES_MINB))
    me_fsbm_split_kernel(const MeParams P) {
  static_assert(S == 32 || S == 64, "half-split ME: S = 32 or 64");
  extern __shared__ __align__(16) uint32_t smem[];
  constexpr int R = S / 2, hi = S - 1 - R;
  constexpr int PW = me_pw(S), CSTRIDE = me_cstride(S);
  uint32_t* cf_s = smem;                                  // 16 rows x 4 words
  uint32_t* win = smem + 64;                              // 4 copies x CSTRIDE words
  uint32_t* red = win + 4 * CSTRIDE;                      // [nwarps][41]

  const int mbx = blockIdx.x, mby = P.row0 + blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t one = (uint32_t)(P.n_rf > 0);            // == 1, opaque (see fadd)
  const int nwarps = blockDim.x >> 5;
  const int h = threadIdx.x & 1;                          // MB half: columns 8h .. 8h+7
  const int off = threadIdx.x >> 1;                       // dx + R
  const uint32_t* wbase = win + (off & 3) * CSTRIDE + (off >> 2) + 2 * h;

  for (int i = threadIdx.x; i < 64; i += blockDim.x)
    cf_s[i] = load4_clamped(P.cf, P.W, P.H, 16 * mbx + 4 * (i & 3), 16 * mby + (i >> 2));

  const int xw0 = 16 * mbx - R, yw0 = 16 * mby - R;
  constexpr int win_rows = S + 15;

  for (int ref = 0; ref < P.n_rf; ++ref) {
    const uint8_t* __restrict__ rf = P.rf[ref];
    __syncthreads();
    {   // a1: 4 byte-shifted copies of the SA window (as me_fsbm_kernel)
      constexpr int chunks = PW >> 2;
      const bool vec_ok = P.vec_ok;
      for (int item = threadIdx.x; item < win_rows * chunks; item += blockDim.x) {
        const int row = item / chunks, k = item - row * chunks;
        const int x = xw0 + 16 * k, y = min(max(yw0 + row, 0), P.H - 1);
        uint32_t w[5];
        if (vec_ok && x >= 0 && x + 20 <= P.W) {
          const uint8_t* src = rf + (size_t)y * P.W + x;
          const uint4 v = __ldg(reinterpret_cast<const uint4*>(src));
          w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
          w[4] = __ldg(reinterpret_cast<const uint32_t*>(src + 16));
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
    __syncthreads();

    uint32_t M[kMesSlots];
#pragma unroll
    for (int s = 0; s < kMesSlots; ++s) M[s] = 0xffffffffu;

    const uint32_t* rank_col = P.rank_tab + off * me_rank_pitch(S) + R;
    uint4 rank_next = __ldg(reinterpret_cast<const uint4*>(rank_col - R));
#pragma unroll 1
    for (int c = 0; c < S; c += kMeT) {
      const int dy0 = -R + c;
      const uint32_t rank[4] = {rank_next.x, rank_next.y, rank_next.z, rank_next.w};
      rank_next = __ldg(reinterpret_cast<const uint4*>(rank_col + min(dy0 + kMeT, hi + 1 - kMeT)));
      const uint32_t* wrow = wbase + (dy0 + R) * PW;

      uint32_t acc[4][2];
      HalfState st[4];
      uint32_t Kp[4][kMesSlots];
      uint2 cfr[16];
#pragma unroll
      for (int i = 0; i < 4 + 15; ++i) {
        if (i < 16) cfr[i] = lds64_v(cf_s + 4 * i + 2 * h);   // CF row i, this half
        const uint32_t w0 = wrow[i * PW], w1 = wrow[i * PW + 1];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const int r = i - t;
          if (r >= 0 && r < 16) {
            acc[t][0] = vad4(cfr[r].x, w0, (r & 3) ? acc[t][0] : 0u);
            acc[t][1] = vad4(cfr[r].y, w1, (r & 3) ? acc[t][1] : 0u);
            if ((r & 3) == 3) {
              const int by = r >> 2;
              if (by == 0) half_row_keys<0>(acc[t], rank[t], st[t], Kp[t], one);
              if (by == 1) half_row_keys<1>(acc[t], rank[t], st[t], Kp[t], one);
              if (by == 2) half_row_keys<2>(acc[t], rank[t], st[t], Kp[t], one);
              if (by == 3) half_row_keys<3>(acc[t], rank[t], st[t], Kp[t], one);
              if (t & 1) {
                if (by == 0) half_fold_pair<0>(M, Kp[t - 1], Kp[t]);
                if (by == 1) half_fold_pair<1>(M, Kp[t - 1], Kp[t]);
                if (by == 2) half_fold_pair<2>(M, Kp[t - 1], Kp[t]);
                if (by == 3) half_fold_pair<3>(M, Kp[t - 1], Kp[t]);
              }
            }
          }
        }
      }
    }

    // a4: per slot, min over the even lanes and over the odd lanes (different partitions)
#pragma unroll
    for (int s = 0; s < kMesSlots; ++s) {
      uint32_t v;
      if (h == 0) v = __reduce_min_sync(0x55555555u, M[s]);
      else v = __reduce_min_sync(0xaaaaaaaau, M[s]);
      if (lane < 2) red[warp * kNPart + mes_part(s, h)] = v;
    }
    __syncthreads();
    for (int p = threadIdx.x; p < kNPart; p += blockDim.x) {
      uint32_t k = red[p];
      for (int w = 1; w < nwarps; ++w) k = min(k, red[w * kNPart + p]);
      const uint32_t mv = __ldg(P.inv_tab + ((k & 0xffffu) >> part_log2n(p)));
      const size_t o = ((size_t)(blockIdx.y * P.mb_cols + mbx) * P.rf_stride + ref) * kNPart + p;
      reinterpret_cast<uint32_t*>(P.out_mvs)[o] = mv;
      P.out_sads[o] = (uint16_t)(k >> 16);
    }
  }
}

}  // namespace feves
