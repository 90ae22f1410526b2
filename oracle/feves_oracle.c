/*
 * feves_oracle.c -- CPU ORACLE for the FEVES inter-prediction hot path
 * (ME -> INT -> SME).  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
 * --impl reference) may load this library.  The product path
 * (paper_conf_icpp_ilicmrs14_b200/) never links, imports or calls it, and it
 * shares no source, header, table or constant generator with csrc/.
 *
 * What it computes, with the passage each function follows
 * (P:<n> = /root/reference/PAPER.md line n; G<k>/O<k> = readings in DESIGN.md §3):
 *
 *   oracle_spiral_rank  G4: tie-break order, built by ENUMERATING the spiral
 *                       (the closed form lives only in the CUDA library).
 *   oracle_ref_px       O0/G5/G6: integer sample with coordinate clamping.
 *   oracle_me           O1, P:6 "The best matching candidate for each
 *                       MB-partition is selected as the one with the minimum
 *                       distortion value ... SAD ... The output of the ME are
 *                       the offsets ... (MVs)".  Every one of the 41
 *                       partitions (P:6 "7 partitioning modes") is computed
 *                       directly from pixels, no 4x4 aggregation.
 *   oracle_sample       O2, P:6 "the RFs are interpolated by applying 6tap and
 *                       linear filters in the Interpolation (INT)"; the filter
 *                       itself is the H.264 luma interpolation the paper
 *                       inherits from JM 18.4, restated in DESIGN.md.
 *   oracle_int_planes   O2, P:6 "Sub-pixel interpolated Frame (SF) structure,
 *                       which size is as large as 16 RFs": 16 phase planes
 *                       built by calling oracle_sample() per sample.
 *   oracle_sme          O3, P:6 "By relying on the MVs from the ME and the SFs
 *                       from the INT, the SME is applied to further refine
 *                       the MVs"; "the MVs from ME define the initial
 *                       search point for the SME".  Uses oracle_sample()
 *                       directly, never the planes.
 *
 * All arithmetic is integer (the paper's 8-bit luma); nothing here is
 * blocked, fused or reordered beyond the definitions above.
 * Parity pins: see tests/test_oracle_*.py (P1..P11 of DESIGN.md §4).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ------------------------------------------------------------------ G7 --
 * The 41 partitions of the 7 modes (P:6), as (ox, oy, w, h) inside the MB.
 * Order (G7): 0: 16x16 | 1-2: 16x8 top,bottom | 3-4: 8x16 left,right |
 * 5-8: 8x8 raster | 9-16: 8x4, 9+2s+k (sub-MB s raster, k=top/bottom) |
 * 17-24: 4x8, 17+2s+k (k=left/right) | 25-40: 4x4, 25+4s+k (raster in s).
 * w = width, h = height (H.264 "WxH" naming).                              */
static void partition_geom(int p, int *ox, int *oy, int *w, int *h)
{
    if (p == 0) { *ox = 0; *oy = 0; *w = 16; *h = 16; return; }
    if (p <= 2) { *ox = 0; *oy = 8 * (p - 1); *w = 16; *h = 8; return; }
    if (p <= 4) { *ox = 8 * (p - 3); *oy = 0; *w = 8; *h = 16; return; }
    if (p <= 8) { int s = p - 5; *ox = 8 * (s % 2); *oy = 8 * (s / 2); *w = 8; *h = 8; return; }
    if (p <= 16) { int s = (p - 9) / 2, k = (p - 9) % 2;
        *ox = 8 * (s % 2); *oy = 8 * (s / 2) + 4 * k; *w = 8; *h = 4; return; }
    if (p <= 24) { int s = (p - 17) / 2, k = (p - 17) % 2;
        *ox = 8 * (s % 2) + 4 * k; *oy = 8 * (s / 2); *w = 4; *h = 8; return; }
    { int s = (p - 25) / 4, k = (p - 25) % 4;
      *ox = 8 * (s % 2) + 4 * (k % 2); *oy = 8 * (s / 2) + 4 * (k / 2); *w = 4; *h = 4; }
}

void oracle_partition_geom(int p, int *out4)
{
    partition_geom(p, &out4[0], &out4[1], &out4[2], &out4[3]);
}

/* ------------------------------------------------------------------ G4 --
 * Spiral order: centre first, then square rings l = 1, 2, ...; inside ring
 * l: for x = -l+1..l-1 take (x,-l) then (x,+l); then for y = -l..l take
 * (-l,y) then (+l,y).  Written as the enumeration, not the closed form.   */
static int spiral_next(int idx, int *dx, int *dy)
{
    /* enumerate positions in order; return position idx */
    if (idx == 0) { *dx = 0; *dy = 0; return 0; }
    int n = 1;
    for (int l = 1;; ++l) {
        for (int x = -l + 1; x <= l - 1; ++x) {
            if (n == idx) { *dx = x; *dy = -l; return 0; } ++n;
            if (n == idx) { *dx = x; *dy = +l; return 0; } ++n;
        }
        for (int y = -l; y <= l; ++y) {
            if (n == idx) { *dx = -l; *dy = y; return 0; } ++n;
            if (n == idx) { *dx = +l; *dy = y; return 0; } ++n;
        }
    }
}

/* Fill order[] with the candidates of the SA in spiral order restricted to
 * [-R, R-1]^2 (G1: S x S candidates, R = S/2); returns how many.          */
static int spiral_candidates(int S, int sa_inclusive, int *odx, int *ody)
{
    int R = S / 2, hi = sa_inclusive ? R : R - 1;
    int want = (R + hi + 1) * (R + hi + 1), n = 0;
    /* every position with max(|x|,|y|) <= R appears before index (2R+1)^2 */
    for (int idx = 0; n < want; ++idx) {
        int x, y;
        spiral_next(idx, &x, &y);
        if (x >= -R && x <= hi && y >= -R && y <= hi) { odx[n] = x; ody[n] = y; ++n; }
    }
    return n;
}

/* the SA's candidates in the order O1 visits them (exported for the key-table test) */
int oracle_spiral_candidates(int S, int sa_inclusive, int *odx, int *ody)
{
    return spiral_candidates(S, sa_inclusive, odx, ody);
}

/* rank of (dx,dy) in the unrestricted spiral, by enumeration (P10 pins it) */
int oracle_spiral_rank(int dx, int dy)
{
    for (int idx = 0;; ++idx) {
        int x, y;
        spiral_next(idx, &x, &y);
        if (x == dx && y == dy) return idx;
    }
}

/* ------------------------------------------------------------- O0/G5/G6 --
 * Pad(F): replicate column W-1 / row H-1 out to Wp, Hp (multiples of 16);
 * ref(x,y) = Pad(F)[clamp(y,0,Hp-1)][clamp(x,0,Wp-1)].  Since the padding
 * replicates the last row/column this equals F[clamp(y,0,H-1)][clamp(x,0,W-1)]. */
static inline int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

static inline int ref_px(const uint8_t *f, int W, int H, int x, int y)
{
    return f[(size_t)clampi(y, 0, H - 1) * W + clampi(x, 0, W - 1)];
}

int oracle_ref_px(const uint8_t *f, int W, int H, int x, int y) { return ref_px(f, W, H, x, y); }

/* CF is sampled the same way (its padding rows/cols replicate, G6). */

/* --------------------------------------------------------------- G18 --
 * Optional rate term (JM-style motion cost; the paper's ME text,
 * P:6, names only the SAD -- lambda = 0 is the default reading G3):
 *   J = SAD + lambda * R(mv),  R(mv) = se(mv.x) + se(mv.y) Exp-Golomb bits of
 *   the quarter-pel MV against the zero predictor (G2: no MV predictor),
 *   se(v): codeNum k = 2v-1 (v > 0) or -2v (v <= 0), bits = 2*floor(log2(k+1)) + 1. */
static int se_bits(int v)
{
    unsigned k = v > 0 ? 2u * (unsigned)v - 1u : 2u * (unsigned)(-v);
    int n = 0;
    while ((k + 1u) >> (n + 1)) ++n;          /* n = floor(log2(k+1)) */
    return 2 * n + 1;
}

int oracle_mv_bits(int qx, int qy) { return se_bits(qx) + se_bits(qy); }

/* ------------------------------------------------------------------ O1 --
 * Integer FSBM ME for the MBs listed in mb_list (indices mby*mb_cols+mbx)
 * over n_rf RFs.  Outputs are written at position i of the list:
 *   out_mvs [n_mb][n_rf][41][2] int16 (dx, dy) full-pel
 *   out_sads[n_mb][n_rf][41]    uint16
 * Returns 0, or -1 on bad arguments.                                      */
/* G21 (SURVEY §8 f4 "predicted-MV centre"): an optional integer-pel MV predictor
 * p per (MB, RF), supplied by the caller (pmv[(mb * n_rf + r) * 2 + {0,1}], mb =
 * the frame MB index mby * mb_cols + mbx; NULL = the zero predictor of G2), each
 * component clamped to [-max_pmv, max_pmv].  The SA is centred on p: candidates
 * mv = p + (dx, dy) over the same (dx, dy) set and spiral order (G1, G4), and the
 * rate term is R(mv - p) on the quarter-pel MV difference, as in JM's motion cost
 * lambda * R(mv - pmv).                                                   */
int oracle_me_pmv(const uint8_t *cf, const uint8_t *const *rfs, int W, int H,
                  int S, int n_rf, int sa_inclusive, int lambda,
                  const int16_t *pmv, int max_pmv,
                  const int32_t *mb_list, int n_mb,
                  int16_t *out_mvs, uint16_t *out_sads, int n_threads);

static int clamp_pmv(const int16_t *pmv, int max_pmv, size_t idx, int comp)
{
    if (!pmv) return 0;
    return clampi(pmv[2 * idx + comp], -max_pmv, max_pmv);
}

int oracle_me_rd(const uint8_t *cf, const uint8_t *const *rfs, int W, int H,
                 int S, int n_rf, int sa_inclusive, int lambda,
                 const int32_t *mb_list, int n_mb,
                 int16_t *out_mvs, uint16_t *out_sads, int n_threads)
{
    return oracle_me_pmv(cf, rfs, W, H, S, n_rf, sa_inclusive, lambda, NULL, 0, mb_list, n_mb,
                         out_mvs, out_sads, n_threads);
}

int oracle_me_pmv(const uint8_t *cf, const uint8_t *const *rfs, int W, int H,
                  int S, int n_rf, int sa_inclusive, int lambda,
                  const int16_t *pmv, int max_pmv,
                  const int32_t *mb_list, int n_mb,
                  int16_t *out_mvs, uint16_t *out_sads, int n_threads)
{
    if (W <= 0 || H <= 0 || S < 2 || (S & 1) || n_rf < 1) return -1;
    int mb_cols = (W + 15) / 16;
    int side = S + (sa_inclusive ? 1 : 0);
    int *cdx = (int *)malloc(sizeof(int) * side * side);
    int *cdy = (int *)malloc(sizeof(int) * side * side);
    int nc = spiral_candidates(S, sa_inclusive, cdx, cdy);
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
    for (int i = 0; i < n_mb; ++i) {
        int mbx = mb_list[i] % mb_cols, mby = mb_list[i] / mb_cols;
        for (int r = 0; r < n_rf; ++r) {
            const uint8_t *rf = rfs[r];
            size_t pi = (size_t)mb_list[i] * n_rf + r;
            int px = clamp_pmv(pmv, max_pmv, pi, 0), py = clamp_pmv(pmv, max_pmv, pi, 1);   /* G21 */
            for (int p = 0; p < 41; ++p) {
                int ox, oy, w, h;
                partition_geom(p, &ox, &oy, &w, &h);
                int x0 = 16 * mbx + ox, y0 = 16 * mby + oy;
                long best = -1, best_sad = 0; int bdx = 0, bdy = 0;
                for (int c = 0; c < nc; ++c) {          /* spiral order, strict < */
                    int dx = px + cdx[c], dy = py + cdy[c];      /* mv = p + SA offset (G21) */
                    long sad = 0;
                    for (int j = 0; j < h; ++j)
                        for (int ii = 0; ii < w; ++ii) {
                            int a = ref_px(cf, W, H, x0 + ii, y0 + j);
                            int b = ref_px(rf, W, H, x0 + ii + dx, y0 + j + dy);
                            sad += a > b ? a - b : b - a;
                        }
                    long cost = sad + (long)lambda * se_bits(4 * (dx - px)) + (long)lambda * se_bits(4 * (dy - py));
                    if (best < 0 || cost < best) { best = cost; best_sad = sad; bdx = dx; bdy = dy; }
                }
                size_t o = ((size_t)i * n_rf + r) * 41 + p;
                out_mvs[2 * o] = (int16_t)bdx; out_mvs[2 * o + 1] = (int16_t)bdy;
                out_sads[o] = (uint16_t)best_sad;
            }
        }
    }
    free(cdx); free(cdy);
    (void)n_threads;
    return 0;
}

int oracle_me(const uint8_t *cf, const uint8_t *const *rfs, int W, int H,
              int S, int n_rf, int sa_inclusive,
              const int32_t *mb_list, int n_mb,
              int16_t *out_mvs, uint16_t *out_sads, int n_threads)
{
    return oracle_me_rd(cf, rfs, W, H, S, n_rf, sa_inclusive, 0, mb_list, n_mb, out_mvs, out_sads, n_threads);
}

/* ------------------------------------------------------------------ O2 --
 * Quarter-pel luma sample of RF f at quarter-pel position (X, Y), i.e.
 * integer position (X>>2, Y>>2) (floor) and phase (X&3, Y&3).  Follows the
 * H.264 luma sample interpolation step by step (DESIGN.md §3 O2):
 *   tap6(p) = p[-2] - 5p[-1] + 20p[0] + 20p[1] - 5p[2] + p[3]
 *   b1 = tap6 horizontal on row y at x-2..x+3,  b = Clip1((b1+16)>>5)
 *   h1 = tap6 vertical on column x at y-2..y+3, h = Clip1((h1+16)>>5)
 *   j1 = tap6 over the vertical b1 values at rows y-2..y+3, j = Clip1((j1+512)>>10)
 *   m = h at column x+1, s = b at row y+1, G,H,M = integer samples at
 *   (x,y),(x+1,y),(x,y+1); quarter samples are (u+v+1)>>1 averages.      */
static inline int clip1(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

static int tap6(int p_m2, int p_m1, int p0, int p1, int p2, int p3)
{
    return p_m2 - 5 * p_m1 + 20 * p0 + 20 * p1 - 5 * p2 + p3;
}

static int b1_at(const uint8_t *f, int W, int H, int x, int y)   /* horizontal half, raw */
{
    return tap6(ref_px(f, W, H, x - 2, y), ref_px(f, W, H, x - 1, y), ref_px(f, W, H, x, y),
                ref_px(f, W, H, x + 1, y), ref_px(f, W, H, x + 2, y), ref_px(f, W, H, x + 3, y));
}

static int h1_at(const uint8_t *f, int W, int H, int x, int y)   /* vertical half, raw */
{
    return tap6(ref_px(f, W, H, x, y - 2), ref_px(f, W, H, x, y - 1), ref_px(f, W, H, x, y),
                ref_px(f, W, H, x, y + 1), ref_px(f, W, H, x, y + 2), ref_px(f, W, H, x, y + 3));
}

static int j1_at(const uint8_t *f, int W, int H, int x, int y)   /* centre half, raw (vertical over b1) */
{
    return tap6(b1_at(f, W, H, x, y - 2), b1_at(f, W, H, x, y - 1), b1_at(f, W, H, x, y),
                b1_at(f, W, H, x, y + 1), b1_at(f, W, H, x, y + 2), b1_at(f, W, H, x, y + 3));
}

/* j computed the other way round (horizontal over h1); P6 pins j1_at == this */
int oracle_j_horizontal_first(const uint8_t *f, int W, int H, int x, int y)
{
    int j1 = tap6(h1_at(f, W, H, x - 2, y), h1_at(f, W, H, x - 1, y), h1_at(f, W, H, x, y),
                  h1_at(f, W, H, x + 1, y), h1_at(f, W, H, x + 2, y), h1_at(f, W, H, x + 3, y));
    return clip1((j1 + 512) >> 10);
}

int oracle_sample(const uint8_t *f, int W, int H, int X, int Y)
{
    int x = X >> 2, y = Y >> 2;          /* arithmetic shift = floor (G10) */
    int xf = X & 3, yf = Y & 3;
    /* the named samples of the standard's figure, each computed only where used */
#define G_ ref_px(f, W, H, x, y)
#define H_ ref_px(f, W, H, x + 1, y)
#define M_ ref_px(f, W, H, x, y + 1)
#define b_ clip1((b1_at(f, W, H, x, y) + 16) >> 5)
#define h_ clip1((h1_at(f, W, H, x, y) + 16) >> 5)
#define m_ clip1((h1_at(f, W, H, x + 1, y) + 16) >> 5)
#define s_ clip1((b1_at(f, W, H, x, y + 1) + 16) >> 5)
#define j_ clip1((j1_at(f, W, H, x, y) + 512) >> 10)
    int v;
    switch (yf * 4 + xf) {                 /* (xFrac, yFrac) -> sample name */
    case 0 * 4 + 0: v = G_; break;                     /* G (0,0) */
    case 0 * 4 + 1: v = (G_ + b_ + 1) >> 1; break;     /* a (1,0) */
    case 0 * 4 + 2: v = b_; break;                     /* b (2,0) */
    case 0 * 4 + 3: v = (H_ + b_ + 1) >> 1; break;     /* c (3,0) */
    case 1 * 4 + 0: v = (G_ + h_ + 1) >> 1; break;     /* d (0,1) */
    case 1 * 4 + 1: v = (b_ + h_ + 1) >> 1; break;     /* e (1,1) */
    case 1 * 4 + 2: v = (b_ + j_ + 1) >> 1; break;     /* f (2,1) */
    case 1 * 4 + 3: v = (b_ + m_ + 1) >> 1; break;     /* g (3,1) */
    case 2 * 4 + 0: v = h_; break;                     /* h (0,2) */
    case 2 * 4 + 1: v = (h_ + j_ + 1) >> 1; break;     /* i (1,2) */
    case 2 * 4 + 2: v = j_; break;                     /* j (2,2) */
    case 2 * 4 + 3: v = (j_ + m_ + 1) >> 1; break;     /* k (3,2) */
    case 3 * 4 + 0: v = (M_ + h_ + 1) >> 1; break;     /* n (0,3) */
    case 3 * 4 + 1: v = (h_ + s_ + 1) >> 1; break;     /* p (1,3) */
    case 3 * 4 + 2: v = (j_ + s_ + 1) >> 1; break;     /* q (2,3) */
    default:        v = (m_ + s_ + 1) >> 1; break;     /* r (3,3) */
    }
#undef G_
#undef H_
#undef M_
#undef b_
#undef h_
#undef m_
#undef s_
#undef j_
    return v;
}

/* raw (pre-clip) intermediates, exposed for the P5 closed-form pins */
int oracle_b1(const uint8_t *f, int W, int H, int x, int y) { return b1_at(f, W, H, x, y); }
int oracle_h1(const uint8_t *f, int W, int H, int x, int y) { return h1_at(f, W, H, x, y); }
int oracle_j1(const uint8_t *f, int W, int H, int x, int y) { return j1_at(f, W, H, x, y); }

/* SF planes (G11): out[phase][row][col], phase = 4*yFrac + xFrac, plane
 * origin at integer position (-pad, -pad), rows/cols as given by the caller.
 * Only rows [row_begin,row_end) of every plane are written.              */
int oracle_int_planes(const uint8_t *f, int W, int H, int pad, int pitch, int rows,
                      int row_begin, int row_end, uint8_t *out, int n_threads)
{
    if (W <= 0 || H <= 0 || pad < 0 || pitch <= 0 || rows <= 0) return -1;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(static)
#endif
    for (int r = row_begin; r < row_end; ++r)
        for (int ph = 0; ph < 16; ++ph)
            for (int c = 0; c < pitch; ++c) {
                int x = c - pad, y = r - pad;
                out[((size_t)ph * rows + r) * pitch + c] =
                    (uint8_t)oracle_sample(f, W, H, 4 * x + (ph & 3), 4 * y + (ph >> 2));
            }
    (void)n_threads;
    return 0;
}

/* ------------------------------------------------------------------ O3 --
 * SME for the MBs in mb_list.  in_mvs/out_qmvs/out_sads are indexed like
 * oracle_me's outputs (position i of the list).  For each (MB, RF, p):
 *   c = 4*mv; best = SADq(c); bestv = c
 *   half:    for k=1..8: v = c + 2*s_k;      if SADq(v) < best: best,bestv = ...
 *   quarter: c' = bestv; for k=1..8: v = c' + s_k; if SADq(v) < best: ...
 * s_k = ring-1 spiral order (0,-1),(0,1),(-1,-1),(1,-1),(-1,0),(1,0),(-1,1),(1,1)
 * SADq(v) = sum over the partition |CF(X,Y) - sample(rf, 4X+v.x, 4Y+v.y)|.   */
static const int ring1[8][2] = { {0,-1},{0,1},{-1,-1},{1,-1},{-1,0},{1,0},{-1,1},{1,1} };

static long sad_q(const uint8_t *cf, const uint8_t *rf, int W, int H,
                  int x0, int y0, int w, int h, int vx, int vy)
{
    long sad = 0;
    for (int j = 0; j < h; ++j)
        for (int i = 0; i < w; ++i) {
            int a = ref_px(cf, W, H, x0 + i, y0 + j);
            int b = oracle_sample(rf, W, H, 4 * (x0 + i) + vx, 4 * (y0 + j) + vy);
            sad += a > b ? a - b : b - a;
        }
    return sad;
}

/* G20 (f4, JM "UseHadamard"): SATD of a partition = sum over its 4x4 blocks of
 * (sum |H D H^T| + 1) >> 1, D = CF - prediction, H = the 4x4 Hadamard matrix.
 * Written as the matrix products (no fast butterfly).                       */
static const int H4[4][4] = { {1, 1, 1, 1}, {1, 1, -1, -1}, {1, -1, -1, 1}, {1, -1, 1, -1} };

static long satd_q(const uint8_t *cf, const uint8_t *rf, int W, int H,
                   int x0, int y0, int w, int h, int vx, int vy)
{
    long total = 0;
    for (int by = 0; by < h; by += 4)
        for (int bx = 0; bx < w; bx += 4) {
            long D[4][4], T[4][4], U[4][4];
            for (int j = 0; j < 4; ++j)
                for (int i = 0; i < 4; ++i) {
                    int X = x0 + bx + i, Y = y0 + by + j;
                    D[j][i] = ref_px(cf, W, H, X, Y) - oracle_sample(rf, W, H, 4 * X + vx, 4 * Y + vy);
                }
            for (int a = 0; a < 4; ++a)            /* T = H D */
                for (int b = 0; b < 4; ++b) {
                    T[a][b] = 0;
                    for (int k = 0; k < 4; ++k) T[a][b] += H4[a][k] * D[k][b];
                }
            for (int a = 0; a < 4; ++a)            /* U = T H^T */
                for (int b = 0; b < 4; ++b) {
                    U[a][b] = 0;
                    for (int k = 0; k < 4; ++k) U[a][b] += T[a][k] * H4[b][k];
                }
            long sum = 0;
            for (int a = 0; a < 4; ++a)
                for (int b = 0; b < 4; ++b) sum += U[a][b] < 0 ? -U[a][b] : U[a][b];
            total += (sum + 1) >> 1;
        }
    return total;
}

long oracle_satd_q(const uint8_t *cf, const uint8_t *rf, int W, int H, int x0, int y0, int w, int h, int vx, int vy)
{
    return satd_q(cf, rf, W, H, x0, y0, w, h, vx, vy);
}

int oracle_sme_ex(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, int lambda, int satd,
                  const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
                  int16_t *out_qmvs, uint16_t *out_sads, int n_threads);

int oracle_sme_rd(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, int lambda,
                  const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
                  int16_t *out_qmvs, uint16_t *out_sads, int n_threads)
{
    return oracle_sme_ex(cf, rfs, W, H, n_rf, lambda, 0, mb_list, n_mb, in_mvs, out_qmvs, out_sads, n_threads);
}

int oracle_sme_pmv(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, int lambda, int satd,
                   const int16_t *pmv, int max_pmv,
                   const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
                   int16_t *out_qmvs, uint16_t *out_sads, int n_threads);

int oracle_sme_ex(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, int lambda, int satd,
                  const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
                  int16_t *out_qmvs, uint16_t *out_sads, int n_threads)
{
    return oracle_sme_pmv(cf, rfs, W, H, n_rf, lambda, satd, NULL, 0, mb_list, n_mb, in_mvs, out_qmvs, out_sads,
                          n_threads);
}

/* metric: SAD (satd = 0, G13) or SATD (satd = 1, G20); outputs the metric value
 * (not the cost J) of the chosen vector.  pmv (G21): rate term R(v - 4p). */
int oracle_sme_pmv(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, int lambda, int satd,
                   const int16_t *pmv, int max_pmv,
                   const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
                   int16_t *out_qmvs, uint16_t *out_sads, int n_threads)
{
    if (W <= 0 || H <= 0 || n_rf < 1) return -1;
    int mb_cols = (W + 15) / 16;
#ifdef _OPENMP
    if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
    for (int i = 0; i < n_mb; ++i) {
        int mbx = mb_list[i] % mb_cols, mby = mb_list[i] / mb_cols;
        for (int r = 0; r < n_rf; ++r)
            for (int p = 0; p < 41; ++p) {
                int ox, oy, w, h;
                partition_geom(p, &ox, &oy, &w, &h);
                int x0 = 16 * mbx + ox, y0 = 16 * mby + oy;
                size_t o = ((size_t)i * n_rf + r) * 41 + p;
                size_t pi = (size_t)mb_list[i] * n_rf + r;
                int qpx = 4 * clamp_pmv(pmv, max_pmv, pi, 0), qpy = 4 * clamp_pmv(pmv, max_pmv, pi, 1);   /* G21 */
                int cx = 4 * in_mvs[2 * o], cy = 4 * in_mvs[2 * o + 1];
                /* cost J = SADq + lambda * R(v) (G18; lambda = 0: pure SAD, G13) */
#define DIST(vx, vy) (satd ? satd_q(cf, rfs[r], W, H, x0, y0, w, h, vx, vy) \
                           : sad_q(cf, rfs[r], W, H, x0, y0, w, h, vx, vy))
                long bsad = DIST(cx, cy);
                long best = bsad + (long)lambda * (se_bits(cx - qpx) + se_bits(cy - qpy));
                int bx = cx, by = cy;
                for (int k = 0; k < 8; ++k) {                     /* half-pel ring */
                    int vx = cx + 2 * ring1[k][0], vy = cy + 2 * ring1[k][1];
                    long s = DIST(vx, vy);
                    long j = s + (long)lambda * (se_bits(vx - qpx) + se_bits(vy - qpy));
                    if (j < best) { best = j; bsad = s; bx = vx; by = vy; }
                }
                int qx = bx, qy = by;
                for (int k = 0; k < 8; ++k) {                     /* quarter-pel ring */
                    int vx = qx + ring1[k][0], vy = qy + ring1[k][1];
                    long s = DIST(vx, vy);
                    long j = s + (long)lambda * (se_bits(vx - qpx) + se_bits(vy - qpy));
                    if (j < best) { best = j; bsad = s; bx = vx; by = vy; }
                }
#undef DIST
                out_qmvs[2 * o] = (int16_t)bx; out_qmvs[2 * o + 1] = (int16_t)by;
                out_sads[o] = (uint16_t)(bsad > 65535 ? 65535 : bsad);   /* SATD can exceed 16 bits (G20) */
            }
    }
    (void)n_threads;
    return 0;
}

int oracle_sme(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf,
               const int32_t *mb_list, int n_mb, const int16_t *in_mvs,
               int16_t *out_qmvs, uint16_t *out_sads, int n_threads)
{
    return oracle_sme_rd(cf, rfs, W, H, n_rf, 0, mb_list, n_mb, in_mvs, out_qmvs, out_sads, n_threads);
}

/* ------------------------------------------------------------------ O4 --
 * Mode decision ("According to the adopted distortion
 * metric and the refined MVs from the SME, the best MB-partitioning mode is
 * selected for each MB").  Per partition and RF: J_p(r) = SAD_p(r) +
 * lambda * R(qmv_p(r)) (G18, from the SME outputs).  H.264 structure (G19):
 *   mb_type 0 16x16: min_r J_0(r)
 *           1 16x8 : sum over p in {1,2} of min_r J_p(r)
 *           2 8x16 : sum over p in {3,4} of min_r J_p(r)
 *           3 P8x8 : sum over sub-MBs s of min over sub_type t in {8x8, 8x4, 4x8,
 *                    4x4} and r of sum over the sub-partitions of J_p(r)
 *                    (one RF per 8x8: sub-8x8 partitions share it)
 * Strict < everywhere, iterating mode, then sub_type, then r in increasing
 * order (lowest index wins ties).  With lambda = 0 the P8x8/4x4 choice never
 * loses (pin P4), so the decision is only informative with a rate term.
 * out[n_mb][10]: mb_type, sub_type[4] (-1 unless P8x8), ref per 8x8 quadrant [4], cost. */
int oracle_mode_decision_pmv(const int16_t *qmvs, const uint16_t *sads, int n_mb, int n_rf, int lambda,
                             const int16_t *pmv, int max_pmv, int32_t *out);

int oracle_mode_decision(const int16_t *qmvs, const uint16_t *sads, int n_mb, int n_rf, int lambda,
                         int32_t *out)
{
    return oracle_mode_decision_pmv(qmvs, sads, n_mb, n_rf, lambda, NULL, 0, out);
}

/* pmv (G21): pmv[(i * n_rf + r) * 2 + {0,1}] for the i-th MB of the arrays; J uses R(qmv - 4p) */
int oracle_mode_decision_pmv(const int16_t *qmvs, const uint16_t *sads, int n_mb, int n_rf, int lambda,
                             const int16_t *pmv, int max_pmv, int32_t *out)
{
    if (n_mb < 0 || n_rf < 1 || n_rf > 16) return -1;
    for (int i = 0; i < n_mb; ++i) {
        long J[16][41];
        for (int r = 0; r < n_rf; ++r)
            for (int p = 0; p < 41; ++p) {
                size_t o = ((size_t)i * n_rf + r) * 41 + p;
                size_t pi = (size_t)i * n_rf + r;
                int qpx = 4 * clamp_pmv(pmv, max_pmv, pi, 0), qpy = 4 * clamp_pmv(pmv, max_pmv, pi, 1);
                J[r][p] = (long)sads[o] + (long)lambda * (se_bits(qmvs[2 * o] - qpx) + se_bits(qmvs[2 * o + 1] - qpy));
            }
        long best = -1; int bt = 0, st[4] = {-1, -1, -1, -1}, rq[4] = {0, 0, 0, 0};
        /* 16x16 */
        { long c = -1; int cr = 0;
          for (int r = 0; r < n_rf; ++r) if (c < 0 || J[r][0] < c) { c = J[r][0]; cr = r; }
          best = c; bt = 0; for (int q = 0; q < 4; ++q) rq[q] = cr; }
        /* 16x8 and 8x16 */
        for (int t = 1; t <= 2; ++t) {
            long c = 0; int pr[2];
            for (int k = 0; k < 2; ++k) {
                int p = (t == 1 ? 1 : 3) + k;
                long m = -1;
                for (int r = 0; r < n_rf; ++r) if (m < 0 || J[r][p] < m) { m = J[r][p]; pr[k] = r; }
                c += m;
            }
            if (c < best) {
                best = c; bt = t;
                if (t == 1) { rq[0] = rq[1] = pr[0]; rq[2] = rq[3] = pr[1]; }
                else        { rq[0] = rq[2] = pr[0]; rq[1] = rq[3] = pr[1]; }
            }
        }
        /* P8x8 */
        { long c = 0; int sst[4], srq[4];
          for (int s = 0; s < 4; ++s) {
              long m = -1;
              for (int t = 0; t < 4; ++t)
                  for (int r = 0; r < n_rf; ++r) {
                      long v;
                      if (t == 0) v = J[r][5 + s];
                      else if (t == 1) v = J[r][9 + 2 * s] + J[r][10 + 2 * s];
                      else if (t == 2) v = J[r][17 + 2 * s] + J[r][18 + 2 * s];
                      else v = J[r][25 + 4 * s] + J[r][26 + 4 * s] + J[r][27 + 4 * s] + J[r][28 + 4 * s];
                      if (m < 0 || v < m) { m = v; sst[s] = t; srq[s] = r; }
                  }
              c += m;
          }
          if (c < best) {
              best = c; bt = 3;
              for (int q = 0; q < 4; ++q) { st[q] = sst[q]; rq[q] = srq[q]; }
          } }
        int32_t *d = out + (size_t)i * 10;
        d[0] = bt;
        for (int q = 0; q < 4; ++q) { d[1 + q] = st[q]; d[5 + q] = rq[q]; }
        d[9] = (int32_t)best;
    }
    return 0;
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
