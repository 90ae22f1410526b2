"""Pins for the predicted-MV centre (G21, SURVEY §8 f4 "lambda*R(MVD) motion cost with a
predicted-MV centre").  CPU only.

P17 known global shift OUTSIDE the SA is recovered exactly (SAD 0) once the predictor points
    near it, and not without it
P18 independent NumPy brute force (tests/np_reference.me_pmv) of the centred, rate-weighted
    search on a textured frame pair with a random predictor field (incl. clamped entries)
P19 flat frames (every SAD 0): the unique rate minimum R(0) puts every ME MV on p and
    keeps every SME MV at 4p; a zero predictor field equals no predictor
P20 translation covariance: centring on p over RF equals the zero-centred search over RF
    translated by p (interior MBs, lambda = 0), MVs shifted by p
"""
import numpy as np
import pytest

import np_reference as npr
from synth import gen_noise, gen_tex


def _field(mbr, mbc, n_rf, seed, lim):
    rng = np.random.default_rng(seed)
    return rng.integers(-lim, lim + 1, (mbr * mbc, n_rf, 2)).astype(np.int16)


def test_p17_shift_outside_sa(orc):
    rng = np.random.default_rng(17)
    rf = rng.integers(0, 256, (64, 80), dtype=np.uint8)
    sx, sy = -7, 5                                   # CF(x, y) = RF(x + sx, y + sy)
    cf = np.roll(rf, (-sy, -sx), axis=(0, 1))
    mbc, mbr = 5, 4
    interior = [1 * mbc + 1, 1 * mbc + 2, 2 * mbc + 2]
    mvs0, sads0 = orc.me(cf, [rf], 8)                # SA [-4, 3]^2: the shift is out of reach
    pm = np.zeros((mbr * mbc, 1, 2), np.int16)
    pm[..., 0], pm[..., 1] = -6, 4                   # predictor near the shift
    mvs, sads = orc.me(cf, [rf], 8, pmv=pm, max_pmv=8)
    for o in interior:
        assert (sads0[o, 0] > 0).all()
        assert (mvs[o, 0] == (sx, sy)).all() and (sads[o, 0] == 0).all()


@pytest.mark.parametrize("lam", [0, 6])
def test_p18_brute_force(orc, lam):
    W, H, S, max_pmv = 48, 32, 8, 3
    rf0, rf1 = gen_tex(W, H, 1, 3), gen_tex(W, H, 2, 3)
    cf = gen_tex(W, H, 0, 3)
    pm = _field(2, 3, 2, 18 + lam, 5)                # some components beyond +-3: clamped
    mvs, sads = orc.me(cf, [rf0, rf1], S, lam=lam, pmv=pm, max_pmv=max_pmv)
    bm, bs = npr.me_pmv(cf, [rf0, rf1], S, lam, pm, max_pmv)
    assert np.array_equal(mvs, bm) and np.array_equal(sads, bs)
    # clamping is part of the reading: the pre-clamped field gives the same result
    mvs_c, sads_c = orc.me(cf, [rf0, rf1], S, lam=lam, pmv=np.clip(pm, -max_pmv, max_pmv), max_pmv=max_pmv)
    assert np.array_equal(mvs, mvs_c) and np.array_equal(sads, sads_c)


def test_p19_flat_frames(orc):
    W, H = 48, 32
    cf = np.full((H, W), 90, np.uint8)
    rf = np.full((H, W), 90, np.uint8)
    pm = _field(2, 3, 1, 19, 4)
    mvs, sads = orc.me(cf, [rf], 16, lam=4, pmv=pm, max_pmv=4)
    assert (sads == 0).all()
    assert np.array_equal(mvs, np.broadcast_to(pm[:, :, None, :], mvs.shape))
    qmvs, qsads = orc.sme(cf, [rf], mvs, lam=4, pmv=pm, max_pmv=4)
    assert (qsads == 0).all() and np.array_equal(qmvs, 4 * mvs)
    z = np.zeros_like(pm)
    for lam in (0, 4):
        a = orc.me(cf, [gen_noise(W, H, 3, 1)], 8, lam=lam)
        b = orc.me(cf, [gen_noise(W, H, 3, 1)], 8, lam=lam, pmv=z, max_pmv=4)
        assert all(np.array_equal(x, y) for x, y in zip(a, b))


def test_p20_translation_covariance(orc):
    W, H, S = 96, 80, 8
    rng = np.random.default_rng(20)
    rf = rng.integers(0, 256, (H, W), dtype=np.uint8)
    cf = gen_tex(W, H, 4, 2)
    px, py = 3, -2
    rf_t = np.roll(rf, (-py, -px), axis=(0, 1))      # rf_t(x, y) = rf(x + px, y + py)
    mbc, mbr = W // 16, H // 16
    pm = np.zeros((mbr * mbc, 1, 2), np.int16)
    pm[..., 0], pm[..., 1] = px, py
    inner = np.array([y * mbc + x for y in range(1, mbr - 1) for x in range(1, mbc - 1)], np.int32)
    a_m, a_s = orc.me(cf, [rf], S, mb_list=inner, pmv=pm, max_pmv=4)
    b_m, b_s = orc.me(cf, [rf_t], S, mb_list=inner)
    assert np.array_equal(a_s, b_s)
    assert np.array_equal(a_m[..., 0], b_m[..., 0] + px) and np.array_equal(a_m[..., 1], b_m[..., 1] + py)


def test_p19_mode_decision_rate_against_predictor(orc):
    # zero distortion, every refined MV on its predictor: every partition costs lam * R(0) = 2 lam,
    # so 16x16 (one partition) wins at cost 2 lam; without the predictor the rate of 4p counts
    n_mb, n_rf, lam = 6, 2, 5
    pm = _field(1, n_mb, n_rf, 21, 6)
    qmvs = np.broadcast_to(4 * pm[:, :, None, :], (n_mb, n_rf, 41, 2)).copy()
    sads = np.zeros((n_mb, n_rf, 41), np.uint16)
    out = orc.mode_decision(qmvs, sads, lam, pmv=pm, max_pmv=6)
    assert (out[:, 0] == 0).all() and (out[:, 9] == 2 * lam).all()
    ref = orc.mode_decision(qmvs, sads, lam)
    exp = [min(lam * (npr.se_bits(4 * pm[i, r, 0]) + npr.se_bits(4 * pm[i, r, 1])) for r in range(n_rf))
           for i in range(n_mb)]
    assert (ref[:, 0] == 0).all() and np.array_equal(ref[:, 9], exp)
