// mode_decision.cuh -- the MC front half: best H.264 P-MB configuration per MB
// (SURVEY §8 f2).  P:29: "According to the adopted distortion metric and the
// refined MVs from the SME, the best MB-partitioning mode is selected for each
// MB in the MC".  Cost per partition and RF (G18): J = SAD + lambda * R(qmv).
// Structure (O4 / G19): 16x16, 16x8, 8x16 with one RF per partition; P8x8 with
// one RF and one sub-type (8x8, 8x4, 4x8, 4x4) per 8x8.  Strict < in the order
// mode, sub-type, RF.  One thread per MB (tiny: reads 41 x n_rf results).
#pragma once
#include "common.cuh"
#include "me_fsbm.cuh"   // se_bits

namespace feves {

struct ModeParams {
  const uint32_t* qmvs;     // [mb][n_rf][41] packed int16 pairs (sme output)
  const uint16_t* sads;
  int32_t* out;             // [mb][10]: mb_type, sub_type[4], ref per 8x8 [4], cost
  int n_mb, n_rf, lambda;   // n_rf = valid RF slots searched (<= rf_stride)
  int rf_stride;            // RF dimension of the layout (the context's n_rf)
  const int16_t* pmv;       // G21 predictor [frame MB][n_rf][2] or null; MB i of the arrays = frame MB mb0 + i
  int max_pmv, mb0;
};

__global__ void __launch_bounds__(128) mode_decision_kernel(const ModeParams P) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_mb) return;
  auto J = [&](int r, int p) -> int {
    const size_t o = ((size_t)i * P.rf_stride + r) * kNPart + p;
    int j = P.sads[o];
    if (P.lambda) {
      const uint32_t mv = P.qmvs[o];
      int qpx = 0, qpy = 0;                  // G21: rate against 4p
      if (P.pmv) {
        const size_t pi = ((size_t)(P.mb0 + i) * P.rf_stride + r) * 2;
        qpx = 4 * min(max((int)P.pmv[pi], -P.max_pmv), P.max_pmv);
        qpy = 4 * min(max((int)P.pmv[pi + 1], -P.max_pmv), P.max_pmv);
      }
      j += P.lambda * (se_bits((int)(int16_t)(mv & 0xffffu) - qpx) + se_bits((int)(int16_t)(mv >> 16) - qpy));
    }
    return j;
  };
  int best, bt = 0, st[4] = {-1, -1, -1, -1}, rq[4];
  {  // 16x16
    int c = J(0, 0), cr = 0;
    for (int r = 1; r < P.n_rf; ++r) { const int v = J(r, 0); if (v < c) { c = v; cr = r; } }
    best = c;
    rq[0] = rq[1] = rq[2] = rq[3] = cr;
  }
  for (int t = 1; t <= 2; ++t) {  // 16x8, 8x16
    int c = 0, pr[2];
    for (int k = 0; k < 2; ++k) {
      const int p = (t == 1 ? 1 : 3) + k;
      int m = J(0, p);
      pr[k] = 0;
      for (int r = 1; r < P.n_rf; ++r) { const int v = J(r, p); if (v < m) { m = v; pr[k] = r; } }
      c += m;
    }
    if (c < best) {
      best = c; bt = t;
      if (t == 1) { rq[0] = rq[1] = pr[0]; rq[2] = rq[3] = pr[1]; }
      else        { rq[0] = rq[2] = pr[0]; rq[1] = rq[3] = pr[1]; }
    }
  }
  {  // P8x8
    int c = 0, sst[4], srq[4];
    for (int s = 0; s < 4; ++s) {
      int m = 0x7fffffff;
      for (int t = 0; t < 4; ++t)
        for (int r = 0; r < P.n_rf; ++r) {
          int v;
          if (t == 0) v = J(r, 5 + s);
          else if (t == 1) v = J(r, 9 + 2 * s) + J(r, 10 + 2 * s);
          else if (t == 2) v = J(r, 17 + 2 * s) + J(r, 18 + 2 * s);
          else v = J(r, 25 + 4 * s) + J(r, 26 + 4 * s) + J(r, 27 + 4 * s) + J(r, 28 + 4 * s);
          if (v < m) { m = v; sst[s] = t; srq[s] = r; }
        }
      c += m;
    }
    if (c < best) {
      best = c; bt = 3;
      for (int q = 0; q < 4; ++q) { st[q] = sst[q]; rq[q] = srq[q]; }
    }
  }
  int32_t* d = P.out + (size_t)i * 10;
  d[0] = bt;
  for (int q = 0; q < 4; ++q) { d[1 + q] = st[q]; d[5 + q] = rq[q]; }
  d[9] = best;
}

}  // namespace feves
