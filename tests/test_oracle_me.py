"""Pins for the ME oracle (O1) and the tie-break (G4).  CPU only.

P1  hand-computed tiny frame (tests/golden/p1_me_tiny.json)
P2  CF == RF -> all SADs 0, all MVs (0,0)
P3  known global integer shift on noise -> exact MV, SAD 0
P4  parent/child monotonicity of minima (sum structure of SAD over 4x4 blocks)
P9  independent NumPy brute force (tests/np_reference.py) on random tiny frames
P10 spiral rank: enumeration (oracle) == closed form (written here); max ranks
"""
import json
import os

import numpy as np
import pytest

import np_reference as npr
from synth import gen_noise, gen_shifted, gen_tex

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def test_p1_hand_computed(orc):
    g = _load("p1_me_tiny.json")
    W, H = g["width"], g["height"]
    x = np.arange(W)
    rf = np.tile(x, (H, 1)).astype(np.uint8)
    cf = np.tile(np.minimum(x + 1, 15), (H, 1)).astype(np.uint8)
    mvs, sads = orc.me(cf, [rf], g["sa_range"])
    for e in g["explicit"]:
        p = e["partition"]
        assert tuple(mvs[0, 0, p]) == tuple(e["mv"]), e
        assert sads[0, 0, p] == e["sad"], e
    # closed form for every partition: SAD = h * (w - [15 in cols]), MV (0,0)
    for p in range(41):
        ox, oy, w, h = orc.partition_geom(p)
        exp = h * (w - (1 if ox <= 15 < ox + w else 0))
        assert sads[0, 0, p] == exp and tuple(mvs[0, 0, p]) == (0, 0), p
    iv = g["inclusive_variant"]
    mvs_i, sads_i = orc.me(cf, [rf], g["sa_range"], sa_inclusive=True)
    assert tuple(mvs_i[0, 0, iv["partition"]]) == tuple(iv["mv"])
    assert sads_i[0, 0, iv["partition"]] == iv["sad"]


@pytest.mark.parametrize("kind", ["tex", "flat", "const"])
def test_p2_identical_frames(orc, kind):
    if kind == "const":
        f = np.full((32, 48), 93, np.uint8)
    elif kind == "flat":
        f = np.zeros((32, 48), np.uint8)
        f[:, 24:] = 200
    else:
        f = gen_tex(48, 32, 0, 5)
    mvs, sads = orc.me(f, [f], 8)
    assert (sads == 0).all()
    assert (mvs == 0).all()


@pytest.mark.parametrize("uv", [(3, -2), (-4, 3), (0, -4), (2, 2)])
def test_p3_global_shift(orc, uv):
    u, v = uv
    S = 8
    rf = gen_noise(64, 48, 0, 21)
    cf = gen_shifted(rf, u, v)
    mvs, sads = orc.me(cf, [rf], S)
    H, W = rf.shape
    mbc = W // 16
    checked = 0
    for o in range(mvs.shape[0]):
        mby, mbx = divmod(o, mbc)
        for p in range(41):
            ox, oy, w, h = orc.partition_geom(p)
            x0, y0 = 16 * mbx + ox + u, 16 * mby + oy + v
            if x0 >= 0 and y0 >= 0 and x0 + w <= W and y0 + h <= H:
                assert tuple(mvs[o, 0, p]) == (u, v), (o, p)
                assert sads[o, 0, p] == 0
                checked += 1
    assert checked > 300


def test_p4_parent_child_minima(orc):
    # SAD(parent, cand) = sum of SAD(children, cand) for every candidate, so the
    # parent's minimum over candidates is >= the sum of the children's minima.
    cf = gen_noise(48, 32, 1, 3)
    rf = gen_noise(48, 32, 0, 3)
    _, s = orc.me(cf, [rf], 8)
    s = s[:, 0].astype(np.int64)
    part4 = lambda sub, k: 25 + 4 * sub + k
    for o in range(s.shape[0]):
        for sub in range(4):
            assert s[o, 5 + sub] >= s[o, 9 + 2 * sub] + s[o, 10 + 2 * sub]       # 8x8 >= 2 x 8x4
            assert s[o, 5 + sub] >= s[o, 17 + 2 * sub] + s[o, 18 + 2 * sub]      # 8x8 >= 2 x 4x8
            assert s[o, 9 + 2 * sub] >= s[o, part4(sub, 0)] + s[o, part4(sub, 1)]
            assert s[o, 10 + 2 * sub] >= s[o, part4(sub, 2)] + s[o, part4(sub, 3)]
            assert s[o, 17 + 2 * sub] >= s[o, part4(sub, 0)] + s[o, part4(sub, 2)]
            assert s[o, 18 + 2 * sub] >= s[o, part4(sub, 1)] + s[o, part4(sub, 3)]
        assert s[o, 1] >= s[o, 5] + s[o, 6] and s[o, 2] >= s[o, 7] + s[o, 8]
        assert s[o, 3] >= s[o, 5] + s[o, 7] and s[o, 4] >= s[o, 6] + s[o, 8]
        assert s[o, 0] >= s[o, 1] + s[o, 2] and s[o, 0] >= s[o, 3] + s[o, 4]


def test_p4_exact_sum_on_single_candidate(orc):
    # With S = 2 but RF constant-shifted so only one candidate can be best... use
    # S such that the SA has exactly one candidate per axis impossible (S>=2);
    # instead check on identical-up-to-noise frames that the 16x16 SAD at a forced
    # common MV equals the sum of its 16 4x4 SADs: when all 41 partitions share
    # the same MV the parent SAD IS the sum of children (not only >=).
    rf = gen_noise(32, 32, 0, 8)
    cf = gen_shifted(rf, 1, 1)
    cf = cf.astype(np.int16)
    cf[5, 5] = (int(cf[5, 5]) + 9) % 256     # small perturbations keep MV (1,1) everywhere
    cf[20, 27] = (int(cf[20, 27]) + 40) % 256
    cf = cf.astype(np.uint8)
    mvs, sads = orc.me(cf, [rf], 4)
    s = sads[:, 0].astype(np.int64)
    for o in range(s.shape[0]):
        if (mvs[o, 0] == mvs[o, 0, 0]).all():
            assert s[o, 0] == s[o, 25:41].sum()
            for sub in range(4):
                assert s[o, 5 + sub] == s[o, 25 + 4 * sub: 29 + 4 * sub].sum()


@pytest.mark.parametrize("seed", range(6))
def test_p9_numpy_bruteforce(orc, seed):
    rng = np.random.default_rng(seed)
    W = int(rng.choice([16, 24, 32, 40]))
    H = int(rng.choice([16, 20, 32]))
    S = int(rng.choice([2, 4, 8]))
    n_rf = int(rng.integers(1, 3))
    kind = seed % 3
    if kind == 0:
        frames = [rng.integers(0, 256, (H, W), dtype=np.uint8) for _ in range(n_rf + 1)]
    elif kind == 1:
        frames = [gen_tex(W, H, t, seed) for t in range(n_rf + 1)]
    else:  # low-entropy content: many ties
        frames = [(rng.integers(0, 3, (H, W)) * 40).astype(np.uint8) for _ in range(n_rf + 1)]
    cf, rfs = frames[-1], frames[:-1][::-1]
    mo, so = orc.me(cf, rfs, S)
    mn, sn = npr.me(cf, rfs, S)
    np.testing.assert_array_equal(so, sn)
    np.testing.assert_array_equal(mo, mn)


def _closed_form(dx, dy):
    l = max(abs(dx), abs(dy))
    if l == 0:
        return 0
    if abs(dy) == l and abs(dx) < l:
        return (2 * l - 1) ** 2 + 2 * (dx + l - 1) + (1 if dy > 0 else 0)
    return (2 * l - 1) ** 2 + 2 * (2 * l - 1) + 2 * (dy + l) + (1 if dx > 0 else 0)


def test_p10_rank_closed_form(orc):
    seen = set()
    for l in range(0, 9):
        for dx in range(-l, l + 1):
            for dy in range(-l, l + 1):
                if max(abs(dx), abs(dy)) != l:
                    continue
                r = orc.spiral_rank(dx, dy)
                assert r == _closed_form(dx, dy), (dx, dy)
                seen.add(r)
    assert seen == set(range(17 * 17))    # a bijection onto 0..(2l+1)^2-1


@pytest.mark.parametrize("S,mx", [(16, 285), (32, 1085), (64, 4221), (128, 16637)])
def test_p10_max_rank(S, mx):
    R = S // 2
    best = max(_closed_form(dx, dy) for dx in range(-R, R) for dy in (-R, R - 1))
    best = max(best, max(_closed_form(dx, dy) for dy in range(-R, R) for dx in (-R, R - 1)))
    assert best == mx and best < 2 ** 16


def test_p10_rank_samples_far(orc):
    for dx, dy in [(-64, -64), (63, 63), (-64, 63), (63, -64), (10, -64), (-64, 5)]:
        assert orc.spiral_rank(dx, dy) == _closed_form(dx, dy)


def test_mb_list_subset_matches_full(orc):
    cf, rf = gen_tex(64, 48, 1, 9), gen_tex(64, 48, 0, 9)
    mv_full, s_full = orc.me(cf, [rf], 8)
    sub = np.array([0, 5, 11], np.int32)
    mv_sub, s_sub = orc.me(cf, [rf], 8, mb_list=sub)
    np.testing.assert_array_equal(mv_sub, mv_full[sub])
    np.testing.assert_array_equal(s_sub, s_full[sub])
