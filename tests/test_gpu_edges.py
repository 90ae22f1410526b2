"""GPU edge cases vs the oracle: degenerate frame sizes, odd widths, 16 RFs,
single-row stripes, stripes in stream mode, repeated contexts."""
import numpy as np
import pytest
import torch

from synth import gen_noise, gen_tex

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def feves():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    return pkg


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _full(feves, orc, cf, rfs, S):
    H, W = cf.shape
    me = feves.MotionEstimator(W, H, S, len(rfs))
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=len(rfs), out_me=me.new_mvs())
    torch.cuda.synchronize()
    n, k = me.mb_rows * me.mb_cols, len(rfs)
    o_m, o_s = orc.me(cf, rfs, S)
    o_q, o_qs = orc.sme(cf, rfs, o_m)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, k, 41), o_s)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, k, 41, 2), o_m)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, k, 41), o_qs)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, k, 41, 2), o_q)
    pad, pitch, rows = orc.sf_layout(W, H, S)
    np.testing.assert_array_equal(sfs[0].cpu().numpy(), orc.int_planes(rfs[0], pad, pitch, rows))
    me.close()


@pytest.mark.parametrize("W,H,S", [(16, 16, 8), (8, 8, 4), (5, 3, 4), (17, 9, 16), (37, 29, 8), (31, 47, 32)])
def test_tiny_and_odd_frames(feves, orc, W, H, S):
    """smaller than one MB, widths not multiple of 4 or 16 (clamped reads, G5/G6)"""
    cf, rf = gen_noise(W, H, 1, W + H), gen_noise(W, H, 0, W + H)
    _full(feves, orc, cf, [rf], S)


def test_sixteen_rfs(feves, orc):
    frames = [gen_tex(32, 32, t, 3) for t in range(17)]
    _full(feves, orc, frames[16], [frames[15 - k] for k in range(16)], 8)


def test_single_row_stripes_stream(feves):
    """stream push with a one-MB-row stripe per 'rank' equals the full-frame stream"""
    W, H, S, n_rf = 64, 80, 16, 2
    frames = [gen_tex(W, H, t, 9) for t in range(4)]
    full = feves.MotionEstimator(W, H, S, n_rf)
    outs = [full.stream_push(_dev(f)) for f in frames]
    torch.cuda.synchronize()
    for r in range(full.mb_rows):
        me = feves.MotionEstimator(W, H, S, n_rf)
        me.set_rows(r, r + 1)
        for t, f in enumerate(frames):
            q, qs, used = me.stream_push(_dev(f))
            torch.cuda.synchronize()
            if used:
                assert torch.equal(q[:, :, :used], outs[t][0][r:r + 1, :, :used])
                assert torch.equal(qs[:, :, :used], outs[t][1][r:r + 1, :, :used])
        me.close()
    full.close()


def test_bad_stripe_and_reset(feves):
    me = feves.MotionEstimator(64, 48, 16, 1)
    with pytest.raises(feves.FevesError):
        me.set_rows(2, 2)
    with pytest.raises(feves.FevesError):
        me.set_rows(0, 4)
    me.stream_reset()
    f = _dev(gen_tex(64, 48, 0, 1))
    _, _, used = me.stream_push(f)
    assert used == 0
    me.close()


def test_many_contexts_and_streams(feves, orc):
    cf, rf = gen_tex(48, 32, 1, 2), gen_tex(48, 32, 0, 2)
    o_m, o_s = orc.me(cf, [rf], 16)
    for i in range(6):
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            me = feves.MotionEstimator(48, 32, 16, 1)
            m, sa = me.estimate(_dev(cf), [_dev(rf)])
        s.synchronize()
        np.testing.assert_array_equal(sa.cpu().numpy().reshape(-1, 1, 41), o_s)
        me.close()


def test_stream_resplit_recomputes_sf(feves):
    """f3: changing the stripe between pushes (as the adaptive split does) keeps results
    identical to the full-frame stream: SFs computed for the old stripe are refreshed."""
    W, H, S, n_rf = 64, 128, 16, 3                      # 8 MB rows
    frames = [gen_tex(W, H, t, 13) for t in range(7)]
    full = feves.MotionEstimator(W, H, S, n_rf)
    ref = [full.stream_push(_dev(f)) for f in frames]
    torch.cuda.synchronize()
    me = feves.MotionEstimator(W, H, S, n_rf)
    splits = [(0, 4), (0, 4), (0, 6), (2, 8), (0, 3), (5, 8), (1, 7)]
    for t, (f, (r0, r1)) in enumerate(zip(frames, splits)):
        me.set_rows(r0, r1)
        q, qs, used = me.stream_push(_dev(f))
        torch.cuda.synchronize()
        if used:
            assert torch.equal(q[:, :, :used], ref[t][0][r0:r1, :, :used]), (t, r0, r1)
            assert torch.equal(qs[:, :, :used], ref[t][1][r0:r1, :, :used]), (t, r0, r1)
    me.close()
    full.close()
