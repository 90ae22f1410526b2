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


def test_single_row_stripes_stream(feves, orc):
    """stream push with a one-MB-row stripe per 'rank': every stripe equals the oracle"""
    W, H, S, n_rf = 64, 80, 16, 2
    frames = [gen_tex(W, H, t, 9) for t in range(4)]
    ref = {t: _oracle_stream(orc, frames, t, n_rf, S) for t in range(1, len(frames))}
    mbc = (W + 15) // 16
    for r in range((H + 15) // 16):
        me = feves.MotionEstimator(W, H, S, n_rf)
        me.set_rows(r, r + 1)
        for t, f in enumerate(frames):
            q, qs, used = me.stream_push(_dev(f))
            torch.cuda.synchronize()
            if used:
                o_q, o_s = ref[t]
                np.testing.assert_array_equal(q.cpu().numpy().reshape(mbc, n_rf, 41, 2)[:, :used],
                                              o_q[r * mbc:(r + 1) * mbc])
                np.testing.assert_array_equal(qs.cpu().numpy().reshape(mbc, n_rf, 41)[:, :used],
                                              o_s[r * mbc:(r + 1) * mbc])
        me.close()


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


def _oracle_stream(orc, frames, t, n_rf, S, rows=None):
    """oracle (qmvs, qsads) of IPPP frame t over its min(t, n_rf) RFs, MB rows [r0, r1)"""
    used = min(t, n_rf)
    H, W = frames[t].shape
    rfs = [frames[t - 1 - k] for k in range(used)]
    mbs = None if rows is None else orc.all_mbs(W, H, rows[0], rows[1])
    o_m, _ = orc.me(frames[t], rfs, S, mb_list=mbs)
    return orc.sme(frames[t], rfs, o_m, mb_list=mbs)


def test_stream_resplit_recomputes_sf(feves, orc):
    """f3: changing the stripe between pushes (as the adaptive split does): every stripe's
    output equals the ORACLE on those MB rows (SFs computed for the old stripe are refreshed)."""
    W, H, S, n_rf = 64, 128, 16, 3                      # 8 MB rows
    frames = [gen_tex(W, H, t, 13) for t in range(7)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    splits = [(0, 4), (0, 4), (0, 6), (2, 8), (0, 3), (5, 8), (1, 7)]
    for t, (f, (r0, r1)) in enumerate(zip(frames, splits)):
        me.set_rows(r0, r1)
        q, qs, used = me.stream_push(_dev(f))
        torch.cuda.synchronize()
        assert used == min(t, n_rf)
        if used:
            o_q, o_s = _oracle_stream(orc, frames, t, n_rf, S, (r0, r1))
            n = (r1 - r0) * me.mb_cols
            np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2)[:, :used], o_q)
            np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41)[:, :used], o_s)
    me.close()


# ---------------------------------------------------------------- ADVICE r01 --

@pytest.mark.parametrize("W,H,S,max_pmv", [(854, 40, 32, 0), (1366, 36, 64, 0), (322, 40, 16, 256),
                                           (320, 48, 16, 256), (101, 37, 8, 40)])
def test_int_border_groups_all_written(feves, orc, W, H, S, max_pmv):
    """INT border path: when W % 4 != 0 (every 16-column group is a border group) or a large
    SF margin (max_pmv) makes more than 32 border groups, EVERY group of every plane is
    written and equals the oracle; SME reading them equals the oracle too."""
    cf, rf = gen_tex(W, H, 1, W + S), gen_tex(W, H, 0, W + S)
    me = feves.MotionEstimator(W, H, S, 1, max_pmv=max_pmv)
    sf = me.new_sf()
    sf.fill_(0xA5)                                      # unwritten bytes would show
    me.interpolate(_dev(rf), out=sf)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(sf.cpu().numpy(), orc.int_planes(rf, me.sf_pad, me.sf_pitch, me.sf_rows))
    if max_pmv:                                         # predictor pointing far right / down reads the margin
        n = me.mb_rows * me.mb_cols
        pm = np.zeros((n, 1, 2), np.int16)
        pm[:, 0, 0] = max_pmv
        pm[::2, 0, 1] = -max_pmv // 3
        me.set_pmv(_dev(pm))
        mvs, sads = me.estimate(_dev(cf), [_dev(rf)])
        q, qs = me.refine(_dev(cf), [sf], mvs, sads)
        torch.cuda.synchronize()
        o_m, o_s = orc.me(cf, [rf], S, pmv=pm, max_pmv=max_pmv)
        np.testing.assert_array_equal(mvs.cpu().numpy().reshape(n, 1, 41, 2), o_m)
        o_q, o_qs = orc.sme(cf, [rf], o_m, pmv=pm, max_pmv=max_pmv)
        np.testing.assert_array_equal(q.cpu().numpy().reshape(n, 1, 41, 2), o_q)
        np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, 1, 41), o_qs)
    else:
        _full(feves, orc, cf, [rf], S)
    me.close()


@pytest.mark.parametrize("S,lam", [(64, 1935), (128, 1731), (16, 2000)])
def test_max_lambda_saturated_sad(feves, orc, S, lam):
    """32-bit ME key J * 2^15 + rank at the largest accepted lambda with saturated SADs (a
    black CF against a white RF, and noise): equals the oracle's 64-bit costs; one more is refused"""
    W, H = 64, 48
    cf = np.zeros((H, W), np.uint8)
    cf[:, W // 2:] = gen_noise(W // 2, H, 0, 5)
    rf = np.full((H, W), 255, np.uint8)
    rf[H // 2:] = gen_noise(W, H - H // 2, 1, 5)
    me = feves.MotionEstimator(W, H, S, 1)
    with pytest.raises(feves.FevesError):
        me.set_lambda(lam + 1)
    me.set_lambda(lam)
    tcf, trf = _dev(cf), [_dev(rf)]
    sfs = [me.new_sf()]
    (m, s), (q, qs) = me.encode_frame(tcf, trf, sfs, n_int=1, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, o_s = orc.me(cf, [rf], S, lam=lam)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, 1, 41, 2), o_m)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, 1, 41), o_s)
    o_q, o_qs = orc.sme(cf, [rf], o_m, lam=lam)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, 1, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, 1, 41), o_qs)
    me.close()


def test_mode_decision_on_the_rf_ramp(feves, orc):
    """me_mode_decision with n_ref = n_ref_used on the first frames of a stream reads only the
    valid RF slots (the others hold garbage here) and equals the oracle's O4 on them"""
    W, H, S, n_rf, lam = 80, 48, 16, 4, 12
    frames = [gen_tex(W, H, t, 29) for t in range(6)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_lambda(lam)
    n = me.mb_rows * me.mb_cols
    for t, f in enumerate(frames):
        qm, qs = me.new_mvs()
        qm.fill_(0)
        qs.fill_(0)                                     # SAD 0 in unused slots would win if read
        qm, qs, used = me.stream_push(_dev(f), out=(qm, qs))
        if not used:
            continue
        modes = me.mode_decision(qm, qs, n_ref=used)
        torch.cuda.synchronize()
        rfs = [frames[t - 1 - k] for k in range(used)]
        o_m, _ = orc.me(f, rfs, S, lam=lam)
        o_q, o_s = orc.sme(f, rfs, o_m, lam=lam)
        np.testing.assert_array_equal(modes.cpu().numpy().reshape(n, 10), orc.mode_decision(o_q, o_s, lam))
        with pytest.raises(feves.FevesError):
            me.mode_decision(qm, qs, n_ref=n_rf + 1)
    me.close()


def test_out_buffers_validated(feves):
    """wrong-size / wrong-kind out= tensors are refused before any device write"""
    me = feves.MotionEstimator(64, 48, 16, 2)
    cf, rf = _dev(gen_tex(64, 48, 1, 3)), _dev(gen_tex(64, 48, 0, 3))
    good = me.new_mvs()
    for bad in [(good[0][:1], good[1]), (good[0], good[1][:, :1]), (good[0].float(), good[1]),
                (good[0].cpu(), good[1].cpu())]:
        with pytest.raises(feves.FevesError):
            me.estimate(cf, [rf, rf], out=bad)
    with pytest.raises(feves.FevesError):                # host outputs must be pinned
        me.stream_push(cf, out=(good[0].cpu(), good[1].cpu()))
    me.close()


def test_misaligned_cf_view(feves, orc):
    """a contiguous CF view at an odd byte offset (W % 4 == 0): no misaligned access, oracle results"""
    W, H, S = 64, 48, 16
    cf, rf = gen_tex(W, H, 1, 8), gen_tex(W, H, 0, 8)
    big = torch.zeros(W * H + 3, dtype=torch.uint8, device="cuda")
    big[1:1 + W * H] = _dev(cf).reshape(-1)
    tcf = big[1:1 + W * H].view(H, W)
    assert tcf.is_contiguous() and tcf.data_ptr() % 4 == 1
    me = feves.MotionEstimator(W, H, S, 1)
    trf = [_dev(rf)]
    sfs = [me.interpolate(trf[0])]
    mvs, sads = me.estimate(tcf, trf)
    q, qs = me.refine(tcf, sfs, mvs, sads)
    torch.cuda.synchronize()
    o_m, o_s = orc.me(cf, [rf], S)
    o_q, o_qs = orc.sme(cf, [rf], o_m)
    n = me.mb_rows * me.mb_cols
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, 1, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, 1, 41), o_qs)
    me.close()


def test_set_stream_own_stream_kept(feves, orc):
    """me_set_stream: a caller stream, then ME_STREAM_OWN (-1) back to the context's own stream
    (kept alive, not destroyed); work stays ordered across the switches"""
    import ctypes
    W, H, S = 48, 32, 16
    cf, rf = gen_tex(W, H, 1, 2), gen_tex(W, H, 0, 2)
    o_m, o_s = orc.me(cf, [rf], S)
    me = feves.MotionEstimator(W, H, S, 1)
    L = feves.lib()
    tcf, trf = _dev(cf), _dev(rf)
    m, s = me.new_mvs()
    torch.cuda.synchronize()
    for k in range(3):
        st = torch.cuda.Stream()
        assert L.me_set_stream(me._ctx, ctypes.c_void_p(st.cuda_stream)) == 0
        assert L.me_estimate(me._ctx, tcf.data_ptr(), (ctypes.c_void_p * 1)(trf.data_ptr()),
                             m.data_ptr(), s.data_ptr()) == 0
        assert L.me_set_stream(me._ctx, ctypes.c_void_p(-1)) == 0
        assert L.me_sync(me._ctx) == 0
        st.synchronize()
        torch.cuda.synchronize()
    assert L.me_estimate(me._ctx, tcf.data_ptr(), (ctypes.c_void_p * 1)(trf.data_ptr()),
                         m.data_ptr(), s.data_ptr()) == 0
    assert L.me_sync(me._ctx) == 0
    n = me.mb_rows * me.mb_cols
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, 1, 41), o_s)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, 1, 41, 2), o_m)
    me.close()


@pytest.mark.parametrize("S", [16, 32, 64, 128, 12])
@pytest.mark.parametrize("rpc", [-1, 0, 1, 2])
def test_rf_per_cta_split(feves, orc, S, rpc):
    """ME_OPT_RF_PER_CTA: the RFs of an MB spread over grid.z CTAs (1 or 2 RFs each, 0 = all in
    one CTA, -1 auto) give the oracle's result for every RF -- compile-time S (incl. the S <= 32 late CF
    store of each CTA's first RF, the S = 128 quadrant keys) and the run-time-S kernel (S = 12), 3 RFs,
    ragged frame"""
    W, H = 72, 40
    frames = [gen_tex(W, H, t, 21 + S) for t in range(4)]
    cf, rfs = frames[3], [frames[2], frames[1], frames[0]]
    me = feves.MotionEstimator(W, H, S, 3)
    me.set_option(me.OPT_RF_PER_CTA, rpc)
    m, s = me.estimate(_dev(cf), [_dev(r) for r in rfs])
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, o_s = orc.me(cf, rfs, S)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, 3, 41), o_s)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, 3, 41, 2), o_m)
    me.close()


@pytest.mark.parametrize("split", [0, 1, 2, 3])
def test_sme_split_modes(feves, orc, split):
    """ME_OPT_SME_SPLIT: every SME work split (one mode, one partition group, or two groups per
    warp, longest tasks dispatched first) gives the oracle's refinement on every partition"""
    W, H, S = 88, 56, 16
    frames = [gen_tex(W, H, t, 5) for t in range(3)]
    cf, rfs = frames[2], [frames[1], frames[0]]
    me = feves.MotionEstimator(W, H, S, 2)
    me.set_option(me.OPT_SME_SPLIT, split)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=2, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, _ = orc.me(cf, rfs, S)
    o_q, o_qs = orc.sme(cf, rfs, o_m)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, 2, 41), o_qs)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, 2, 41, 2), o_q)
    me.close()


def test_scheduling_option_values(feves):
    """ME_OPT_RF_PER_CTA accepts -1 (auto) .. 16, ME_OPT_SME_SPLIT 0 .. 3; anything else is
    ME_EINVAL and leaves the context usable"""
    me = feves.MotionEstimator(32, 32, 16, 2)
    for v in (-1, 0, 1, 16):
        me.set_option(me.OPT_RF_PER_CTA, v)
    for v in (0, 1, 2, 3):
        me.set_option(me.OPT_SME_SPLIT, v)
    for opt, bad in ((me.OPT_RF_PER_CTA, -2), (me.OPT_RF_PER_CTA, 17), (me.OPT_SME_SPLIT, -1), (me.OPT_SME_SPLIT, 4)):
        with pytest.raises(feves.FevesError):
            me.set_option(opt, bad)
    f = _dev(gen_tex(32, 32, 1, 2))
    me.estimate(f, [f, f])                    # still usable
    torch.cuda.synchronize()
    me.close()
