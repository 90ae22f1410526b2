"""Pins for the rate term (G18) and mode decision (O4, §8 f2).  CPU only.

P12 hand-computed: se(v) bit lengths; the P1 frame with an inclusive SA under lambda
    = 0 / 10 / 100 moves the 16x16 MV (1,-1) -> (1,0) -> (0,0) exactly at the
    thresholds derived by hand
P13 independent NumPy brute force (tests/np_reference.py): RD-ME and an explicit
    enumeration of every H.264 P-MB configuration for the mode decision
P14 closed forms for the mode decision (zero residual, crafted tables, ties, refs)
"""
import numpy as np
import pytest

import np_reference as npr
from synth import gen_noise, gen_tex


@pytest.mark.parametrize("v,bits", [(0, 1), (1, 3), (-1, 3), (2, 5), (-2, 5), (3, 5), (4, 7), (-4, 7), (7, 7),
                                    (8, 9), (-8, 9), (64, 15)])
def test_p12_exp_golomb_bits(orc, v, bits):
    assert orc.mv_bits(v, 0) == bits + 1          # + se(0) = 1 bit for the other component
    assert npr.se_bits(v) == bits


@pytest.mark.parametrize("lam,mv,sad", [(0, (1, -1), 0), (10, (1, 0), 0), (39, (1, 0), 0), (41, (0, 0), 240),
                                        (100, (0, 0), 240)])
def test_p12_rate_moves_the_mv(orc, lam, mv, sad):
    # P1 frame: RF(x,y)=x, CF(x,y)=min(x+1,15), SA {-1,0,1}^2 (inclusive).  16x16 SADs:
    # dx=+1 -> 0, dx=0 -> 240, dx=-1 -> 480 (RF constant along y).  Costs (quarter-pel MVs):
    # J(1,0)=8*lam, J(1,+-1)=14*lam, J(0,0)=240+2*lam -> (1,0) beats (0,0) iff lam < 40.
    x = np.arange(16)
    rf = np.tile(x, (16, 1)).astype(np.uint8)
    cf = np.tile(np.minimum(x + 1, 15), (16, 1)).astype(np.uint8)
    mvs, sads = orc.me(cf, [rf], 2, sa_inclusive=True, lam=lam)
    assert tuple(mvs[0, 0, 0]) == mv and sads[0, 0, 0] == sad


def test_p12_large_lambda_forces_zero_mv(orc):
    rf = gen_noise(48, 32, 0, 4)
    cf = gen_noise(48, 32, 1, 4)
    mvs, _ = orc.me(cf, [rf], 8, lam=100000)
    assert (mvs == 0).all()
    q, _ = orc.sme(cf, [rf], mvs, lam=100000)
    assert (q == 0).all()


@pytest.mark.parametrize("seed,lam", [(0, 4), (1, 20), (2, 2)])
def test_p13_rd_me_vs_numpy(orc, seed, lam):
    rng = np.random.default_rng(seed)
    frames = [gen_tex(32, 32, t, seed) for t in range(3)] if seed != 1 else \
        [rng.integers(0, 256, (32, 24), dtype=np.uint8) for _ in range(3)]
    cf, rfs = frames[2], [frames[1], frames[0]]
    mo, so = orc.me(cf, rfs, 8, lam=lam)
    mn, sn = npr.me_rd(cf, rfs, 8, lam)
    np.testing.assert_array_equal(mo, mn)
    np.testing.assert_array_equal(so, sn)


@pytest.mark.parametrize("seed,lam,n_rf", [(0, 0, 1), (1, 6, 2), (2, 30, 2), (3, 2, 3)])
def test_p13_mode_decision_vs_enumeration(orc, seed, lam, n_rf):
    rng = np.random.default_rng(seed)
    n = 6
    qmvs = rng.integers(-9, 10, (n, n_rf, 41, 2)).astype(np.int16)
    sads = rng.integers(0, 400, (n, n_rf, 41)).astype(np.uint16)
    if seed % 2 == 0:                      # also exercise exact ties
        sads[:, :, 25:] = sads[:, :, 25:] // 100 * 100
    np.testing.assert_array_equal(orc.mode_decision(qmvs, sads, lam), npr.mode_decision(qmvs, sads, lam))


def test_p14_zero_residual_prefers_fewest_mvs(orc):
    qmvs = np.zeros((1, 1, 41, 2), np.int16)
    sads = np.zeros((1, 1, 41), np.uint16)
    out = orc.mode_decision(qmvs, sads, 5)
    assert out[0].tolist() == [0, -1, -1, -1, -1, 0, 0, 0, 0, 10]    # 16x16, cost 2 bits * 5


def test_p14_crafted_16x8(orc):
    s = np.zeros((1, 1, 41), np.uint16)
    s[0, 0, 0], s[0, 0, 1:3], s[0, 0, 3:5] = 100, 10, 60
    s[0, 0, 5:9], s[0, 0, 9:25], s[0, 0, 25:41] = 30, 15, 8
    out = orc.mode_decision(np.zeros((1, 1, 41, 2), np.int16), s, 0)
    assert out[0, 0] == 1 and out[0, 9] == 20


def test_p14_ties_and_refs(orc):
    s = np.full((1, 2, 41), 500, np.uint16)
    s[0, :, 0] = 40
    s[0, :, 1:3] = 20                        # 16x16 ties 16x8 (40 == 20+20) -> 16x16 (lower mode)
    s[0, 1, 0] = 40                          # equal across refs -> ref 0
    out = orc.mode_decision(np.zeros((1, 2, 41, 2), np.int16), s, 0)
    assert out[0, 0] == 0 and out[0, 5:9].tolist() == [0, 0, 0, 0]
    s[0, 1, 0] = 39                          # ref 1 now strictly better
    out = orc.mode_decision(np.zeros((1, 2, 41, 2), np.int16), s, 0)
    assert out[0, 0] == 0 and out[0, 5:9].tolist() == [1, 1, 1, 1] and out[0, 9] == 39


def test_p14_lambda0_never_beats_finest(orc):
    # with lam = 0 the P8x8/4x4 configuration (one RF per 8x8) bounds the decision from above
    cf, rfs = gen_tex(48, 32, 2, 5), [gen_tex(48, 32, 1, 5), gen_tex(48, 32, 0, 5)]
    mvs, _ = orc.me(cf, rfs, 8)
    q, s = orc.sme(cf, rfs, mvs)
    out = orc.mode_decision(q, s, 0)
    for i in range(out.shape[0]):
        finest = sum(int(s[i, :, 25 + 4 * b:29 + 4 * b].astype(np.int64).sum(axis=1).min()) for b in range(4))
        assert out[i, 9] <= finest


# ------------------------------------------------------------------ P15: SATD --

def test_p15_satd_closed_forms(orc):
    # D constant c on a 4x4 block: H D H^T has only the DC term 16c -> (16|c| + 1) >> 1 = 8|c|
    rf = np.full((16, 16), 100, np.uint8)
    for c in (0, 1, 7, -5):
        cf = np.full((16, 16), 100 + c, np.uint8)
        assert orc.satd_q(cf, rf, 0, 0, 4, 4, 0, 0) == 8 * abs(c)
        assert orc.satd_q(cf, rf, 0, 0, 16, 16, 0, 0) == 16 * 8 * abs(c)       # 16 blocks
    # single impulse d in a block: every coefficient is +-d -> (16|d| + 1) >> 1 = 8|d|
    cf = rf.copy()
    cf[1, 2] = 100 + 9
    assert orc.satd_q(cf, rf, 0, 0, 4, 4, 0, 0) == 72
    # odd total: one coefficient pattern giving sum 2k+1 is impossible for integer D (all
    # coefficients share parity), so (s+1)>>1 == s/2 here; a 2-pixel difference d,-d in one row
    cf = rf.copy()
    cf[0, 0], cf[0, 1] = 103, 97            # D row 0 = (3, -3, 0, 0)
    assert orc.satd_q(cf, rf, 0, 0, 4, 4, 0, 0) == (sum(abs(v) for v in (0, 0, 6, 6)) * 4 + 1) // 2


def test_p15_satd_sme_vs_numpy(orc):
    cf, rf0 = gen_tex(32, 32, 1, 8), gen_tex(32, 32, 0, 8)
    mvs, _ = orc.me(cf, [rf0], 8)
    qo, so = orc.sme(cf, [rf0], mvs, satd=True)
    qn, sn = npr.sme_satd(cf, [rf0], mvs, 8)
    np.testing.assert_array_equal(qo, qn)
    np.testing.assert_array_equal(so, sn)
    qo2, so2 = orc.sme(cf, [rf0], mvs, satd=True, lam=5)
    qn2, sn2 = npr.sme_satd(cf, [rf0], mvs, 8, lam=5)
    np.testing.assert_array_equal(qo2, qn2)
    np.testing.assert_array_equal(so2, sn2)
