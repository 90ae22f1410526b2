"""Pins for the INT oracle (O2) and the SME oracle (O3).  CPU only.

P5  closed forms: constant plane, step edge, impulse, ramp (tests/golden/p5_*.json)
P6  j vertical-first == j horizontal-first; 1-D content: j == b
P7  each quarter plane == rounded average of its two named neighbour planes
P8  SME invariants + half-pel synthetic shift
P9  independent NumPy planes / SME (tests/np_reference.py)
"""
import json
import os

import numpy as np
import pytest

import np_reference as npr
from synth import gen_noise, gen_tex

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold():
    with open(os.path.join(GOLD, "p5_int_closed_forms.json")) as f:
        return json.load(f)


def test_p5_constant(orc):
    c = _gold()["constant"]["c"]
    f = np.full((24, 40), c, np.uint8)
    pad, pitch, rows = orc.sf_layout(40, 24, 8)
    P = orc.int_planes(f, pad, pitch, rows)
    assert (P == c).all()


@pytest.mark.parametrize("which", ["step", "impulse"])
def test_p5_edge_and_impulse(orc, which):
    g = _gold()[which]
    k = g["k"]
    row = np.zeros(24, np.uint8)
    if which == "step":
        row[k:] = 255
    else:
        row[k] = 255
    f = np.tile(row, (8, 1))
    for off, b1, b in zip(g["x_offsets"], g["b1"], g["b"]):
        assert orc.raw("b1", f, k + off, 3) == b1
        assert orc.sample(f, 4 * (k + off) + 2, 4 * 3) == b     # phase (2,0) = b


def test_p5_ramp(orc):
    a = _gold()["ramp"]["alpha"]
    W = 80
    f = np.tile((a * np.arange(W)).astype(np.uint8), (8, 1))
    for x in range(3, W - 4):
        assert orc.sample(f, 4 * x + 2, 8) == (32 * a * x + 16 * a + 16) >> 5


def test_p6_j_both_orders(orc):
    f = gen_noise(24, 20, 0, 4)
    for y in range(-3, 23, 3):
        for x in range(-3, 27, 2):
            assert orc.sample(f, 4 * x + 2, 4 * y + 2) == orc.raw("j_hfirst", f, x, y)


def test_p6_1d_content_j_equals_b(orc):
    row = gen_noise(32, 1, 0, 6)[0]
    f = np.tile(row, (12, 1))
    for x in range(-2, 34):
        assert orc.sample(f, 4 * x + 2, 4 * 5 + 2) == orc.sample(f, 4 * x + 2, 4 * 5)


def test_p7_quarter_identities(orc):
    f = gen_tex(40, 24, 0, 12)
    pad, pitch, rows = orc.sf_layout(40, 24, 8)
    P = orc.int_planes(f, pad, pitch, rows).astype(np.int32)
    avg = lambda u, v: (u + v + 1) >> 1
    ph = lambda xf, yf: P[4 * yf + xf]
    right = lambda A: A[:, 1:]        # value at x+1
    down = lambda A: A[1:, :]         # value at y+1
    c0 = lambda A: A[:, :-1]
    r0 = lambda A: A[:-1, :]
    G, b, h, j = ph(0, 0), ph(2, 0), ph(0, 2), ph(2, 2)
    np.testing.assert_array_equal(ph(1, 0), avg(G, b))                              # a
    np.testing.assert_array_equal(c0(ph(3, 0)), avg(right(G), c0(b)))               # c
    np.testing.assert_array_equal(ph(0, 1), avg(G, h))                              # d
    np.testing.assert_array_equal(r0(ph(0, 3)), avg(down(G), r0(h)))                # n
    np.testing.assert_array_equal(ph(2, 1), avg(b, j))                              # f
    np.testing.assert_array_equal(ph(1, 2), avg(h, j))                              # i
    np.testing.assert_array_equal(c0(ph(3, 2)), avg(c0(j), right(h)))               # k: m = h at x+1
    np.testing.assert_array_equal(r0(ph(2, 3)), avg(r0(j), down(b)))                # q: s = b at y+1
    np.testing.assert_array_equal(ph(1, 1), avg(b, h))                              # e
    np.testing.assert_array_equal(c0(ph(3, 1)), avg(c0(b), right(h)))               # g
    np.testing.assert_array_equal(r0(ph(1, 3)), avg(r0(h), down(b)))                # p
    np.testing.assert_array_equal(r0(c0(ph(3, 3))), avg(r0(right(h)), c0(down(b))))  # r


@pytest.mark.parametrize("seed", range(4))
def test_p9_planes_vs_numpy(orc, seed):
    rng = np.random.default_rng(100 + seed)
    W, H = int(rng.choice([16, 24, 40])), int(rng.choice([16, 20, 36]))
    f = rng.integers(0, 256, (H, W), dtype=np.uint8) if seed % 2 else gen_tex(W, H, 0, seed)
    pad, pitch, rows = orc.sf_layout(W, H, 8)
    np.testing.assert_array_equal(orc.int_planes(f, pad, pitch, rows), npr.planes(f, pad, pitch, rows))


def test_int_plane_row_subset(orc):
    f = gen_tex(32, 32, 0, 1)
    pad, pitch, rows = orc.sf_layout(32, 32, 8)
    full = orc.int_planes(f, pad, pitch, rows)
    part = orc.int_planes(f, pad, pitch, rows, row_begin=10, row_end=30)
    np.testing.assert_array_equal(part[:, 10:30], full[:, 10:30])
    assert (part[:, :10] == 0).all()


# ------------------------------------------------------------------ SME ----

def _me_sme(orc, cf, rfs, S):
    mvs, sads = orc.me(cf, rfs, S)
    qmvs, qs = orc.sme(cf, rfs, mvs)
    return mvs, sads, qmvs, qs


def test_p2_sme_identical(orc):
    f = gen_tex(48, 32, 0, 2)
    mvs, sads, qmvs, qs = _me_sme(orc, f, [f], 8)
    assert (qs == 0).all() and (qmvs == 0).all()


@pytest.mark.parametrize("seed", range(3))
def test_p8_invariants(orc, seed):
    cf, rf0, rf1 = gen_tex(48, 32, 2, seed), gen_tex(48, 32, 1, seed), gen_tex(48, 32, 0, seed)
    mvs, sads, qmvs, qs = _me_sme(orc, cf, [rf0, rf1], 8)
    assert (qs <= sads).all()
    d = qmvs.astype(np.int32) - 4 * mvs.astype(np.int32)
    assert np.abs(d).max() <= 3
    # centre SAD equals the ME SAD: with no improvement the qmv stays 4*mv and SAD equal
    same = (d == 0).all(-1)
    assert (qs[same] == sads[same]).all()
    # tex content moving at (1.25, -0.75) px/frame gives strictly better sub-pel SADs
    assert qs.astype(np.int64).sum() < sads.astype(np.int64).sum()


@pytest.mark.parametrize("uv", [(1, 0), (-2, 1)])
def test_p8_half_pel_synthetic(orc, uv):
    u, v = uv
    W, H = 48, 32
    rf = gen_tex(W, H, 0, 31)
    # CF(x, y) = b-plane sample of RF at integer (x+u, y+v), i.e. quarter position (4(x+u)+2, 4(y+v))
    cf = np.array([[orc.sample(rf, 4 * (x + u) + 2, 4 * (y + v)) for x in range(W)] for y in range(H)],
                  np.uint8)
    mvs, sads, qmvs, qs = _me_sme(orc, cf, [rf], 8)
    mbc = W // 16
    hit = 0
    for o in range(qmvs.shape[0]):
        mby, mbx = divmod(o, mbc)
        for p in range(41):
            ox, oy, w, h = orc.partition_geom(p)
            x0, y0 = 16 * mbx + ox, 16 * mby + oy
            interior = x0 + u - 3 >= 0 and y0 + v - 3 >= 0 and x0 + w + u + 4 <= W and y0 + h + v + 4 <= H
            if interior and qs[o, 0, p] == 0:
                assert tuple(qmvs[o, 0, p]) == (4 * u + 2, 4 * v)
                hit += 1
    assert hit >= 20


@pytest.mark.parametrize("seed", range(3))
def test_p9_sme_vs_numpy(orc, seed):
    rng = np.random.default_rng(200 + seed)
    W, H, S = 32, 32, 4
    frames = [gen_tex(W, H, t, seed) for t in range(3)] if seed != 1 else \
        [rng.integers(0, 256, (H, W), dtype=np.uint8) for _ in range(3)]
    cf, rfs = frames[2], [frames[1], frames[0]]
    mvs, _ = orc.me(cf, rfs, S)
    qo, so = orc.sme(cf, rfs, mvs)
    qn, sn = npr.sme(cf, rfs, mvs, S)
    np.testing.assert_array_equal(so, sn)
    np.testing.assert_array_equal(qo, qn)


def test_sme_subset_matches_full(orc):
    cf, rf = gen_tex(48, 32, 1, 4), gen_tex(48, 32, 0, 4)
    mvs, _ = orc.me(cf, [rf], 8)
    q_full, s_full = orc.sme(cf, [rf], mvs)
    sub = np.array([1, 4], np.int32)
    q_sub, s_sub = orc.sme(cf, [rf], mvs[sub], mb_list=sub)
    np.testing.assert_array_equal(q_sub, q_full[sub])
    np.testing.assert_array_equal(s_sub, s_full[sub])
