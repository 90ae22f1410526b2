"""P11: MB-row stripes are independent given an R+3-row halo.

ME, INT and SME for MB row r read CF rows [16r, 16r+15] and RF rows
[16r-R-3, 16r+15+R+3] only (clamped).  So running the oracle on a stripe whose
frames are CORRUPTED outside that window must give exactly the full-frame
result restricted to the stripe.  This is what makes the multi-GPU split exact.
"""
import numpy as np
import pytest

from synth import gen_tex


def stripes(n_rows, g):
    base, extra = divmod(n_rows, g)
    out, r0 = [], 0
    for i in range(g):
        r1 = r0 + base + (1 if i < extra else 0)
        out.append((r0, r1))
        r0 = r1
    return out


def corrupt_outside(f, y_lo, y_hi, seed):
    f = f.copy()
    rng = np.random.default_rng(seed)
    H = f.shape[0]
    lo, hi = max(0, y_lo), min(H, y_hi)
    f[:lo] = rng.integers(0, 256, f[:lo].shape, dtype=np.uint8)
    f[hi:] = rng.integers(0, 256, f[hi:].shape, dtype=np.uint8)
    return f


@pytest.mark.parametrize("g", [2, 3, 4])
def test_p11_stripe_equivalence(orc, g):
    W, H, S = 48, 88, 8          # 6 MB rows, last row ragged (88 = 5*16 + 8)
    R = S // 2
    cf = gen_tex(W, H, 2, 77)
    rfs = [gen_tex(W, H, 1, 77), gen_tex(W, H, 0, 77)]
    mbc, mbr = W // 16, -(-H // 16)
    mv_full, s_full = orc.me(cf, rfs, S)
    q_full, qs_full = orc.sme(cf, rfs, mv_full)
    for k, (r0, r1) in enumerate(stripes(mbr, g)):
        lo, hi = 16 * r0 - R - 3, 16 * r1 + R + 3
        cf_s = corrupt_outside(cf, 16 * r0, 16 * r1, 10 + k)
        rfs_s = [corrupt_outside(rf, lo, hi, 20 + k + i) for i, rf in enumerate(rfs)]
        mbs = np.arange(r0 * mbc, r1 * mbc, dtype=np.int32)
        mv, s = orc.me(cf_s, rfs_s, S, mb_list=mbs)
        np.testing.assert_array_equal(mv, mv_full[mbs])
        np.testing.assert_array_equal(s, s_full[mbs])
        q, qs = orc.sme(cf_s, rfs_s, mv, mb_list=mbs)
        np.testing.assert_array_equal(q, q_full[mbs])
        np.testing.assert_array_equal(qs, qs_full[mbs])
