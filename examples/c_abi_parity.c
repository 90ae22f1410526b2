/*
 * c_abi_parity.c -- uses include/feves_me.h from plain C (no Python, no torch):
 * me_create -> int_interpolate -> me_estimate -> sme_refine on a seeded frame
 * pair, then compares every MV / SAD / SF byte with the CPU oracle
 * (oracle/liboracle.so, test infrastructure).  Exit 0 = bit-exact.
 *
 *   gcc -O2 -I include -o c_abi_parity examples/c_abi_parity.c \
 *       -L paper_conf_icpp_ilicmrs14_b200 -lfeves_me -L oracle -loracle \
 *       -L /usr/local/cuda/lib64 -lcudart
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <cuda_runtime_api.h>

#include "feves_me.h"

/* oracle (oracle/feves_oracle.c) */
int oracle_me(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int S, int n_rf, int sa_inclusive,
              const int32_t *mb_list, int n_mb, int16_t *out_mvs, uint16_t *out_sads, int n_threads);
int oracle_sme(const uint8_t *cf, const uint8_t *const *rfs, int W, int H, int n_rf, const int32_t *mb_list,
               int n_mb, const int16_t *in_mvs, int16_t *out_qmvs, uint16_t *out_sads, int n_threads);
int oracle_int_planes(const uint8_t *f, int W, int H, int pad, int pitch, int rows, int row_begin, int row_end,
                      uint8_t *out, int n_threads);

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
    fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_)); return 2; } } while (0)
#define ME(x) do { int s_ = (x); if (s_ != ME_OK) { fprintf(stderr, "%s: %s\n", #x, me_strerror(s_)); return 3; } } while (0)

static uint32_t lcg = 12345;
static uint8_t rnd(void) { lcg = lcg * 1103515245u + 12345u; return (uint8_t)(lcg >> 16); }

int main(void) {
    const int W = 100, H = 72, S = 16, NRF = 2;          /* ragged: 7 x 5 MBs */
    const size_t fb = (size_t)W * H;
    uint8_t *h_f[3];
    for (int k = 0; k < 3; ++k) {                        /* smooth-ish content moving right */
        h_f[k] = (uint8_t *)malloc(fb);
        for (int y = 0; y < H; ++y)
            for (int x = 0; x < W; ++x)
                h_f[k][y * W + x] = (uint8_t)(((x + 2 * k) * 7 + y * 3) % 200 + (rnd() & 15));
    }
    const uint8_t *cf = h_f[2];
    const uint8_t *rf_h[2] = {h_f[1], h_f[0]};           /* ref_idx 0 = most recent */

    me_ctx *ctx = me_create(W, H, S, NRF);
    if (!ctx) { fprintf(stderr, "me_create: %s\n", me_strerror(me_last_error())); return 4; }
    int mbc, mbr, pad, pitch, rows;
    ME(me_get_layout(ctx, &mbc, &mbr, &pad, &pitch, &rows));
    const int nmb = mbc * mbr;
    const size_t nmv = (size_t)nmb * NRF * ME_N_PART, sfb = (size_t)ME_N_PHASE * rows * pitch;

    uint8_t *d_cf, *d_rf[2], *d_sf[2];
    int16_t *d_mv, *d_qmv;
    uint16_t *d_sad, *d_qsad;
    CK(cudaMalloc((void **)&d_cf, fb));
    CK(cudaMemcpy(d_cf, cf, fb, cudaMemcpyHostToDevice));
    for (int k = 0; k < NRF; ++k) {
        CK(cudaMalloc((void **)&d_rf[k], fb));
        CK(cudaMalloc((void **)&d_sf[k], sfb));
        CK(cudaMemcpy(d_rf[k], rf_h[k], fb, cudaMemcpyHostToDevice));
    }
    CK(cudaMalloc((void **)&d_mv, nmv * 4));
    CK(cudaMalloc((void **)&d_qmv, nmv * 4));
    CK(cudaMalloc((void **)&d_sad, nmv * 2));
    CK(cudaMalloc((void **)&d_qsad, nmv * 2));

    /* host pointers are rejected before anything is enqueued */
    if (me_estimate(ctx, cf, (const uint8_t *const *)d_rf, d_mv, d_sad) != ME_EINVAL) { fprintf(stderr, "host ptr accepted\n"); return 5; }

    for (int k = 0; k < NRF; ++k) ME(int_interpolate(ctx, d_rf[k], d_sf[k]));
    ME(me_estimate(ctx, d_cf, (const uint8_t *const *)d_rf, d_mv, d_sad));
    ME(sme_refine(ctx, d_cf, (const uint8_t *const *)d_sf, d_mv, d_sad, d_qmv, d_qsad));
    ME(me_sync(ctx));

    int16_t *g_mv = malloc(nmv * 4), *g_qmv = malloc(nmv * 4), *o_mv = malloc(nmv * 4), *o_qmv = malloc(nmv * 4);
    uint16_t *g_sad = malloc(nmv * 2), *g_qsad = malloc(nmv * 2), *o_sad = malloc(nmv * 2), *o_qsad = malloc(nmv * 2);
    uint8_t *g_sf = malloc(sfb), *o_sf = malloc(sfb);
    CK(cudaMemcpy(g_mv, d_mv, nmv * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(g_sad, d_sad, nmv * 2, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(g_qmv, d_qmv, nmv * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(g_qsad, d_qsad, nmv * 2, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(g_sf, d_sf[0], sfb, cudaMemcpyDeviceToHost));

    int32_t *mbs = malloc(sizeof(int32_t) * nmb);
    for (int i = 0; i < nmb; ++i) mbs[i] = i;
    oracle_me(cf, rf_h, W, H, S, NRF, 0, mbs, nmb, o_mv, o_sad, 0);
    oracle_sme(cf, rf_h, W, H, NRF, mbs, nmb, o_mv, o_qmv, o_qsad, 0);
    oracle_int_planes(rf_h[0], W, H, pad, pitch, rows, 0, rows, o_sf, 0);

    int bad = 0;
    bad += memcmp(g_mv, o_mv, nmv * 4) != 0;
    bad += memcmp(g_sad, o_sad, nmv * 2) != 0;
    bad += memcmp(g_qmv, o_qmv, nmv * 4) != 0;
    bad += memcmp(g_qsad, o_qsad, nmv * 2) != 0;
    bad += memcmp(g_sf, o_sf, sfb) != 0;
    printf("c_abi_parity: %d MBs x %d RFs x 41 partitions, SF %zu bytes: %s\n", nmb, NRF, sfb,
           bad ? "MISMATCH" : "bit-exact");
    me_destroy(ctx);
    return bad ? 1 : 0;
}
