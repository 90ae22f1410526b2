"""GPU parity for the predicted-MV centre (G21): the CUDA path through the C-ABI
vs the oracle, bit-exact -- ME (runtime-S kernel, window origin per (MB, RF)), SME and the mode
decision with the rate measured against the predictor, the per-RF pipelined launches (the
predictor pointer offset per RF), the IPPP stream, and predictors beyond the clamp."""
import numpy as np
import pytest
import torch

from synth import gen_noise, gen_tex

pytestmark = pytest.mark.gpu

GEN = {"tex": gen_tex, "noise": gen_noise}


@pytest.fixture(scope="module")
def feves():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    assert torch.cuda.is_available()
    return pkg


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _field(n_mb, n_rf, seed, lim):
    rng = np.random.default_rng(seed)
    f = rng.integers(-lim, lim + 1, (n_mb, n_rf, 2)).astype(np.int16)
    f[0, 0] = (16, -16)                              # 16-aligned window origin (vector staging) when in range
    return f


@pytest.mark.parametrize("W,H,S,n_rf,max_pmv,lam,kind,pipeline,satd", [
    (80, 48, 16, 2, 6, 0, "tex", 0, 0),
    (80, 48, 16, 2, 6, 7, "tex", 0, 0),
    (128, 64, 32, 2, 16, 0, "noise", 0, 0),          # R = 16: vector staging for 16-aligned predictors
    (128, 64, 32, 3, 16, 12, "tex", 1, 0),           # per-RF pipelined ME/SME launches
    (70, 40, 8, 2, 5, 30, "noise", 0, 0),            # ragged frame
    (96, 48, 64, 1, 8, 3, "tex", 0, 0),
    (80, 48, 16, 2, 6, 5, "tex", 0, 1),              # SATD in SME
])
def test_pmv_me_sme_mode_decision(feves, orc, W, H, S, n_rf, max_pmv, lam, kind, pipeline, satd):
    g = GEN[kind]
    cf = g(W, H, n_rf, 7 + S)
    rfs = [g(W, H, n_rf - 1 - k, 7 + S) for k in range(n_rf)]
    me = feves.MotionEstimator(W, H, S, n_rf, max_pmv=max_pmv)
    n = me.mb_rows * me.mb_cols
    pm = _field(n, n_rf, 100 + S + lam, max_pmv + 3)  # some components beyond the clamp
    tpm = _dev(pm)
    me.set_pmv(tpm)
    if lam:
        me.set_lambda(lam)
    if pipeline:
        me.set_option(me.OPT_PIPELINE_RF, 1)
    if satd:
        me.set_sme_satd(True)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    modes = me.mode_decision(q, qs)
    torch.cuda.synchronize()
    o_m, o_s = orc.me(cf, rfs, S, lam=lam, pmv=pm, max_pmv=max_pmv)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, n_rf, 41, 2), o_m)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, n_rf, 41), o_s)
    o_q, o_qs = orc.sme(cf, rfs, o_m, lam=lam, satd=bool(satd), pmv=pm, max_pmv=max_pmv)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_qs)
    if lam:
        np.testing.assert_array_equal(modes.cpu().numpy().reshape(n, 10),
                                      orc.mode_decision(o_q, o_qs, lam, pmv=pm, max_pmv=max_pmv))
    # no predictor on the same context: the zero-centred search
    me.set_pmv(None)
    (m0, s0), _ = me.encode_frame(tcf, trfs, sfs, n_int=0, out_me=me.new_mvs())
    torch.cuda.synchronize()
    o_m0, o_s0 = orc.me(cf, rfs, S, lam=lam)
    np.testing.assert_array_equal(m0.cpu().numpy().reshape(n, n_rf, 41, 2), o_m0)
    np.testing.assert_array_equal(s0.cpu().numpy().reshape(n, n_rf, 41), o_s0)
    me.close()


def test_pmv_recovers_shift_outside_sa(feves):
    W, H, S = 96, 64, 16
    rng = np.random.default_rng(5)
    rf = rng.integers(0, 256, (H, W), dtype=np.uint8)
    sx, sy = 13, -11                                 # beyond the SA [-8, 7]
    cf = np.roll(rf, (-sy, -sx), axis=(0, 1))
    me = feves.MotionEstimator(W, H, S, 1, max_pmv=16)
    n = me.mb_rows * me.mb_cols
    pm = np.zeros((n, 1, 2), np.int16)
    pm[..., 0], pm[..., 1] = 10, -9
    me.set_pmv(_dev(pm))
    (m, s), _ = me.encode_frame(_dev(cf), [_dev(rf)], [me.new_sf()], n_int=1, out_me=me.new_mvs())
    torch.cuda.synchronize()
    m = m.cpu().numpy().reshape(me.mb_rows, me.mb_cols, 41, 2)
    s = s.cpu().numpy().reshape(me.mb_rows, me.mb_cols, 41)
    inner = (slice(1, me.mb_rows - 1), slice(1, me.mb_cols - 1))
    assert (m[inner][..., 0] == sx).all() and (m[inner][..., 1] == sy).all() and (s[inner] == 0).all()
    me.close()


def test_pmv_stream_push(feves, orc):
    """IPPP stream with a predictor field: RF r of push t is frame t-1-r (ring order)."""
    W, H, S, n_rf, max_pmv, lam = 80, 48, 16, 2, 4, 6
    frames = [gen_tex(W, H, t, 71) for t in range(4)]
    me = feves.MotionEstimator(W, H, S, n_rf, max_pmv=max_pmv)
    me.set_lambda(lam)
    n = me.mb_rows * me.mb_cols
    pm = _field(n, n_rf, 9, max_pmv)
    me.set_pmv(_dev(pm))
    for t, f in enumerate(frames):
        qm, qs, used = me.stream_push(_dev(f))
        torch.cuda.synchronize()
        if used == 0:
            continue
        rfs = [frames[t - 1 - k] for k in range(used)]
        sub = np.ascontiguousarray(pm[:, :used])
        o_m, _ = orc.me(f, rfs, S, lam=lam, pmv=sub, max_pmv=max_pmv)
        o_q, o_s = orc.sme(f, rfs, o_m, lam=lam, pmv=sub, max_pmv=max_pmv)
        np.testing.assert_array_equal(qm.cpu().numpy().reshape(n, n_rf, 41, 2)[:, :used], o_q)
        np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41)[:, :used], o_s)
    me.close()


def test_set_pmv_needs_room(feves):
    me = feves.MotionEstimator(64, 48, 16, 1)
    with pytest.raises(feves.FevesError):
        me.set_pmv(torch.zeros((12, 1, 2), dtype=torch.int16, device="cuda"))
    me.close()


@pytest.mark.parametrize("halo_only", [0, 1])
def test_pmv_stripes_stream(feves, orc, halo_only):
    """Predictor on MB-row stripes (the ranks of a sharded run): every stripe's stream push,
    with only the stripe + (R + max_pmv) halo rows copied when halo_only, == the oracle."""
    W, H, S, n_rf, max_pmv, lam = 96, 112, 16, 2, 12, 3   # 7 MB rows
    frames = [gen_tex(W, H, t, 81) for t in range(4)]
    me = feves.MotionEstimator(W, H, S, n_rf, max_pmv=max_pmv)
    me.set_lambda(lam)
    me.set_option(me.OPT_HALO_ONLY, halo_only)
    n = me.mb_rows * me.mb_cols
    pm = _field(n, n_rf, 13, max_pmv)
    pm[:, :, 1] = np.where(np.arange(n)[:, None] % 2 == 0, max_pmv, -max_pmv)   # reach the full halo
    me.set_pmv(_dev(pm))
    for r0, r1 in [(0, 3), (3, 5), (5, 7)]:
        me.set_rows(r0, r1)
        me.stream_reset()
        mbs = np.arange(r0 * me.mb_cols, r1 * me.mb_cols, dtype=np.int32)
        for t, f in enumerate(frames):
            qm, qs, used = me.stream_push(_dev(f))
            torch.cuda.synchronize()
            if used == 0:
                continue
            rfs = [frames[t - 1 - k] for k in range(used)]
            sub = np.ascontiguousarray(pm[:, :used])
            o_m, _ = orc.me(f, rfs, S, mb_list=mbs, lam=lam, pmv=sub, max_pmv=max_pmv)
            o_q, o_s = orc.sme(f, rfs, o_m, mb_list=mbs, lam=lam, pmv=sub, max_pmv=max_pmv)
            k = len(mbs)
            np.testing.assert_array_equal(qm.cpu().numpy().reshape(k, n_rf, 41, 2)[:, :used], o_q)
            np.testing.assert_array_equal(qs.cpu().numpy().reshape(k, n_rf, 41)[:, :used], o_s)
    me.close()


def test_pmv_full_size_sampled(feves, orc):
    """BASELINE config[2] size (1080p, 4 RF, S 64) with the rate term and a predictor field
    (synthetic motion + seeded jitter, some beyond the clamp) through encode_frame, the
    launch configuration bench.py --lam 4 --max-pmv 8 times; sampled MBs vs the oracle."""
    from synth import CONFIGS, make_workload
    from test_gpu_parity import _sample_mbs
    cfg, lam, max_pmv = CONFIGS["1080p_sa64_4rf"], 4, 8
    cf, rfs = make_workload(cfg, kind="tex")
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf, max_pmv=max_pmv)
    me.set_lambda(lam)
    n = me.mb_rows * me.mb_cols
    rng = np.random.default_rng(64)
    pm = rng.integers(-3, 4, (n, cfg.n_rf, 2)).astype(np.int16)
    for r in range(cfg.n_rf):
        pm[:, r, 0] += round(-1.25 * (r + 1))
        pm[:, r, 1] += round(0.75 * (r + 1))
    pm[::97] = 11                                        # beyond the clamp
    me.set_pmv(_dev(pm))
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (mvs, sads), (qmvs, qsads) = me.encode_frame(tcf, trfs, sfs, n_int=cfg.n_rf, out_me=me.new_mvs())
    torch.cuda.synchronize()
    mvs = mvs.cpu().numpy().reshape(n, cfg.n_rf, 41, 2)
    sads = sads.cpu().numpy().reshape(n, cfg.n_rf, 41)
    qmvs = qmvs.cpu().numpy().reshape(n, cfg.n_rf, 41, 2)
    qsads = qsads.cpu().numpy().reshape(n, cfg.n_rf, 41)
    mbs = np.union1d(_sample_mbs(me.mb_cols, me.mb_rows, 8, 6), np.arange(0, n, 97 * 20, dtype=np.int32))
    o_m, o_s = orc.me(cf, rfs, cfg.sa_range, mb_list=mbs, lam=lam, pmv=pm, max_pmv=max_pmv)
    np.testing.assert_array_equal(mvs[mbs], o_m)
    np.testing.assert_array_equal(sads[mbs], o_s)
    o_q, o_qs = orc.sme(cf, rfs, o_m, mb_list=mbs, lam=lam, pmv=pm, max_pmv=max_pmv)
    np.testing.assert_array_equal(qmvs[mbs], o_q)
    np.testing.assert_array_equal(qsads[mbs], o_qs)
    # everywhere: every ME MV lies in its clamped predictor's SA
    p = np.clip(pm, -max_pmv, max_pmv)[:, :, None, :].astype(np.int32)
    d = mvs.astype(np.int32) - p
    assert (d >= -cfg.sa_range // 2).all() and (d < cfg.sa_range // 2).all()
    me.close()
