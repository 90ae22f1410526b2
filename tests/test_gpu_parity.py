"""GPU parity: the CUDA path (through the C-ABI) vs the CPU oracle, element by element.

Bar: bit-exact (all arithmetic on the path is integer).  MVs are unique under
G4/G14, so MVs and SADs are compared exactly.  Small cases run the oracle on
the whole frame (several MBs, ragged right/bottom edges, several SA sizes);
BASELINE.json's full sizes compare sampled MBs (corners, edges, stripe rows,
seeded random rows) in the same launch configuration bench.py times.
"""
import numpy as np
import pytest
import torch

from synth import CONFIGS, gen_flat, gen_noise, gen_shifted, gen_tex, make_workload

pytestmark = pytest.mark.gpu

GEN = {"tex": gen_tex, "noise": gen_noise, "flat": gen_flat}


@pytest.fixture(scope="module")
def feves():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    assert torch.cuda.is_available()
    return pkg


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _frames(kind, W, H, n_rf, seed):
    g = GEN[kind]
    cf = g(W, H, n_rf, seed)
    rfs = [g(W, H, n_rf - 1 - k, seed) for k in range(n_rf)]
    return cf, rfs


def _run_me(feves, cf, rfs, S):
    H, W = cf.shape
    me = feves.MotionEstimator(W, H, S, len(rfs))
    mvs, sads = me.estimate(_dev(cf), [_dev(r) for r in rfs])
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    out = mvs.cpu().numpy().reshape(n, len(rfs), 41, 2), sads.cpu().numpy().reshape(n, len(rfs), 41)
    me.close()
    return out


SMALL = [  # (W, H, S, n_rf, kind)
    (64, 48, 16, 1, "tex"), (64, 48, 16, 2, "noise"), (80, 40, 8, 1, "flat"),
    (72, 52, 32, 2, "tex"),            # ragged: 72 = 4.5 MBs, 52 = 3.25 MBs
    (100, 36, 4, 3, "noise"), (50, 30, 6, 1, "tex"), (96, 80, 64, 1, "tex"),
    (48, 48, 12, 2, "flat"), (40, 40, 128, 1, "noise"),
    # runtime-S kernel where the last staged word of a window row is read (PW == (S-1)/4 + 4)
    (70, 50, 18, 1, "noise"), (96, 70, 66, 1, "noise"),
]


@pytest.mark.parametrize("W,H,S,n_rf,kind", SMALL)
def test_me_full_frame_small(feves, orc, W, H, S, n_rf, kind):
    cf, rfs = _frames(kind, W, H, n_rf, 1000 + W + S)
    g_mvs, g_sads = _run_me(feves, cf, rfs, S)
    o_mvs, o_sads = orc.me(cf, rfs, S)
    np.testing.assert_array_equal(g_sads, o_sads)
    np.testing.assert_array_equal(g_mvs, o_mvs)


@pytest.mark.parametrize("kind", ["tex", "noise", "flat"])
def test_me_cif_config(feves, orc, kind):
    """BASELINE config 1: CIF 352x288, 2 frames, 1 RF, SA 16, full frame."""
    cfg = CONFIGS["cif"]
    cf, rfs = make_workload(cfg, kind=kind)
    g_mvs, g_sads = _run_me(feves, cf, rfs, cfg.sa_range)
    o_mvs, o_sads = orc.me(cf, rfs, cfg.sa_range)
    np.testing.assert_array_equal(g_sads, o_sads)
    np.testing.assert_array_equal(g_mvs, o_mvs)


@pytest.mark.parametrize("uv", [(5, -3), (-8, 7)])
def test_me_global_shift(feves, uv):
    rf = gen_noise(128, 96, 0, 3)
    cf = gen_shifted(rf, *uv)
    g_mvs, g_sads = _run_me(feves, cf, [rf], 16)
    interior = g_mvs.reshape(6, 8, 1, 41, 2)[1:-1, 1:-1]
    assert (interior[..., 0] == uv[0]).all() and (interior[..., 1] == uv[1]).all()


def test_me_identical_frames(feves):
    f = gen_flat(96, 64, 0, 9)
    g_mvs, g_sads = _run_me(feves, f, [f, f], 32)
    assert (g_sads == 0).all() and (g_mvs == 0).all()


@pytest.mark.parametrize("W,H,S", [(64, 48, 8), (72, 52, 16), (50, 30, 64), (33, 17, 128)])
def test_int_planes_full(feves, orc, W, H, S):
    rf = gen_noise(W, H, 0, W * H) if S != 16 else gen_tex(W, H, 0, 5)
    me = feves.MotionEstimator(W, H, S, 1)
    sf = me.interpolate(_dev(rf))
    torch.cuda.synchronize()
    pad, pitch, rows = orc.sf_layout(W, H, S)
    assert (me.sf_pad, me.sf_pitch, me.sf_rows) == (pad, pitch, rows)
    np.testing.assert_array_equal(sf.cpu().numpy(), orc.int_planes(rf, pad, pitch, rows))
    me.close()


@pytest.mark.parametrize("W,H,S,n_rf,kind", [(64, 48, 16, 2, "tex"), (72, 52, 8, 1, "noise"),
                                             (80, 48, 32, 2, "flat"), (50, 30, 64, 1, "tex")])
def test_sme_full_frame(feves, orc, W, H, S, n_rf, kind):
    cf, rfs = _frames(kind, W, H, n_rf, 7 + S)
    me = feves.MotionEstimator(W, H, S, n_rf)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.interpolate(r) for r in trfs]
    mvs, sads = me.estimate(tcf, trfs)
    q1, s1 = me.refine(tcf, sfs, mvs, sads)
    q2, s2 = me.refine(tcf, sfs, mvs, None)          # centre recomputed from the SF
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_mvs, _ = orc.me(cf, rfs, S)
    o_q, o_s = orc.sme(cf, rfs, o_mvs)
    np.testing.assert_array_equal(mvs.cpu().numpy().reshape(n, n_rf, 41, 2), o_mvs)
    for q, s in ((q1, s1), (q2, s2)):
        np.testing.assert_array_equal(s.cpu().numpy().reshape(n, n_rf, 41), o_s)
        np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    me.close()


def test_encode_frame_equals_separate_calls(feves):
    W, H, S = 96, 64, 16
    cf, rfs = _frames("tex", W, H, 2, 4)
    me = feves.MotionEstimator(W, H, S, 2)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs_a = [me.interpolate(r) for r in trfs]
    mvs, sads = me.estimate(tcf, trfs)
    qa, sa = me.refine(tcf, sfs_a, mvs, sads)
    sfs_b = [me.new_sf() for _ in trfs]
    me.set_fused(True)
    (m2, s2), (qb, sb) = me.encode_frame(tcf, trfs, sfs_b, n_int=2, out_me=me.new_mvs())
    assert me.launches == 2 + 1              # one INT launch per RF, fused ME+SME
    me.set_fused(False)
    sfs_c = [me.new_sf() for _ in trfs]
    (m3, s3), (qc, sc) = me.encode_frame(tcf, trfs, sfs_c, n_int=2, out_me=me.new_mvs())
    assert me.launches == 2 + 2              # ... ME, SME as separate launches
    torch.cuda.synchronize()
    assert torch.equal(mvs, m2) and torch.equal(sads, s2) and torch.equal(qa, qb) and torch.equal(sa, sb)
    assert torch.equal(mvs, m3) and torch.equal(sads, s3) and torch.equal(qa, qc) and torch.equal(sa, sc)
    for a, b, c in zip(sfs_a, sfs_b, sfs_c):
        assert torch.equal(a, b) and torch.equal(a, c)
    me.close()


@pytest.mark.parametrize("fused,S", [(True, 32), (False, 32), (True, 128), (False, 128)])
def test_stream_fused_and_unfused_agree(feves, orc, fused, S):
    W, H, n_rf = 96, 64, 2
    frames = [gen_noise(W, H, t, 17) for t in range(4)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_fused(fused)
    for f in frames:
        qm, qs, used = me.stream_push(_dev(f))
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    rfs = [frames[2], frames[1]]
    o_mvs, _ = orc.me(frames[3], rfs, S)
    o_q, o_s = orc.sme(frames[3], rfs, o_mvs)
    np.testing.assert_array_equal(qm.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_s)
    me.close()


def test_host_pointer_rejected(feves):
    me = feves.MotionEstimator(64, 48, 16, 1)
    cf = torch.zeros(48, 64, dtype=torch.uint8)          # host tensor
    with pytest.raises(feves.FevesError):
        me.estimate(cf, [cf])
    me.close()


# ----------------------------------------------------- full BASELINE sizes --

def _sample_mbs(mb_cols, mb_rows, n_random, seed, stripes=(2, 4, 8)):
    rows = {0, mb_rows - 1}
    for g in stripes:
        base, extra = divmod(mb_rows, g)
        r = 0
        for i in range(g):
            r += base + (1 if i < extra else 0)
            rows |= {min(r, mb_rows - 1), max(r - 1, 0)}
    rng = np.random.default_rng(seed)
    mbs = {0, mb_cols - 1, (mb_rows - 1) * mb_cols, mb_rows * mb_cols - 1}
    for r in rows:
        mbs |= {r * mb_cols, r * mb_cols + mb_cols - 1, r * mb_cols + int(rng.integers(mb_cols))}
    mbs |= set(int(v) for v in rng.integers(0, mb_rows * mb_cols, n_random))
    return np.array(sorted(mbs), np.int32)


@pytest.mark.parametrize("name,n_random", [("1080p_sa32", 24), ("1080p_sa64_4rf", 12), ("2160p_sa128", 3)])
def test_full_size_sampled(feves, orc, name, n_random):
    """Full BASELINE sizes through encode_frame (the launch bench.py times); sampled MBs."""
    cfg = CONFIGS[name]
    cf, rfs = make_workload(cfg, kind="tex")
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (mvs, sads), (qmvs, qsads) = me.encode_frame(tcf, trfs, sfs, n_int=cfg.n_rf, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    mvs = mvs.cpu().numpy().reshape(n, cfg.n_rf, 41, 2)
    sads = sads.cpu().numpy().reshape(n, cfg.n_rf, 41)
    qmvs = qmvs.cpu().numpy().reshape(n, cfg.n_rf, 41, 2)
    qsads = qsads.cpu().numpy().reshape(n, cfg.n_rf, 41)
    mbs = _sample_mbs(me.mb_cols, me.mb_rows, n_random, 5)
    if name == "2160p_sa128":
        mbs = mbs[np.random.default_rng(1).choice(len(mbs), 10, replace=False)]
    o_mvs, o_sads = orc.me(cf, rfs, cfg.sa_range, mb_list=mbs)
    np.testing.assert_array_equal(sads[mbs], o_sads)
    np.testing.assert_array_equal(mvs[mbs], o_mvs)
    o_q, o_qs = orc.sme(cf, rfs, o_mvs, mb_list=mbs)
    np.testing.assert_array_equal(qsads[mbs], o_qs)
    np.testing.assert_array_equal(qmvs[mbs], o_q)
    # properties that hold everywhere
    assert (qsads <= sads).all()
    assert np.abs(qmvs.astype(np.int32) - 4 * mvs.astype(np.int32)).max() <= 3
    # INT: sampled rows of the first SF (top margin, frame edge rows, bottom margin)
    pad, pitch, rows = orc.sf_layout(cfg.width, cfg.height, cfg.sa_range)
    sf0 = sfs[0].cpu().numpy()
    for r in (0, pad - 1, pad, pad + cfg.height // 2, pad + cfg.height - 1, rows - 1):
        ref = orc.int_planes(rfs[0], pad, pitch, rows, row_begin=r, row_end=r + 1)
        np.testing.assert_array_equal(sf0[:, r], ref[:, r])
    me.close()


@pytest.mark.parametrize("kind", ["tex", "flat", "noise"])
def test_full_frame_1080p_s64_every_mb(feves, orc, kind):
    """1080p, SA 64x64 (the bench's ME kernel), 1 RF: EVERY MB's 41 MVs/SADs (ME and SME) and the
    whole SF equal the oracle -- not a sample (the oracle takes ~10 s on the box's cores)."""
    cfg = CONFIGS["1080p_sa64_4rf"]
    cf, rfs = make_workload(cfg, kind=kind)
    rfs = rfs[:1]
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, 1)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf()]
    (mvs, sads), (qmvs, qsads) = me.encode_frame(tcf, trfs, sfs, n_int=1, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_mvs, o_sads = orc.me(cf, rfs, cfg.sa_range)
    np.testing.assert_array_equal(sads.cpu().numpy().reshape(n, 1, 41), o_sads)
    np.testing.assert_array_equal(mvs.cpu().numpy().reshape(n, 1, 41, 2), o_mvs)
    o_q, o_qs = orc.sme(cf, rfs, o_mvs)
    np.testing.assert_array_equal(qsads.cpu().numpy().reshape(n, 1, 41), o_qs)
    np.testing.assert_array_equal(qmvs.cpu().numpy().reshape(n, 1, 41, 2), o_q)
    if kind == "tex":
        pad, pitch, rows = orc.sf_layout(cfg.width, cfg.height, cfg.sa_range)
        np.testing.assert_array_equal(sfs[0].cpu().numpy(), orc.int_planes(rfs[0], pad, pitch, rows))
    me.close()


def test_2160p_s128_every_mb_of_three_rows(feves, orc):
    """2160p, SA 128x128 (quadrant key-sum, half-window staging), 1 RF: every MB of the top,
    middle and bottom MB rows (720 MBs incl. both frame corners) equals the oracle, ME and SME."""
    cfg = CONFIGS["2160p_sa128"]
    cf, rfs = make_workload(cfg, kind="tex")
    rfs = rfs[:1]
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, 1)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf()]
    (mvs, sads), (qmvs, qsads) = me.encode_frame(tcf, trfs, sfs, n_int=1, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    rows = (0, me.mb_rows // 2, me.mb_rows - 1)
    mbs = np.array([r * me.mb_cols + c for r in rows for c in range(me.mb_cols)], np.int32)
    o_mvs, o_sads = orc.me(cf, rfs, cfg.sa_range, mb_list=mbs)
    np.testing.assert_array_equal(sads.cpu().numpy().reshape(n, 1, 41)[mbs], o_sads)
    np.testing.assert_array_equal(mvs.cpu().numpy().reshape(n, 1, 41, 2)[mbs], o_mvs)
    o_q, o_qs = orc.sme(cf, rfs, o_mvs, mb_list=mbs)
    np.testing.assert_array_equal(qsads.cpu().numpy().reshape(n, 1, 41)[mbs], o_qs)
    np.testing.assert_array_equal(qmvs.cpu().numpy().reshape(n, 1, 41, 2)[mbs], o_q)
    me.close()


def test_determinism(feves):
    cfg = CONFIGS["1080p_sa32"]
    cf, rfs = make_workload(cfg, kind="flat")
    a = _run_me(feves, cf, rfs, cfg.sa_range)
    b = _run_me(feves, cf, rfs, cfg.sa_range)
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[1], b[1])


@pytest.mark.parametrize("g", [2, 3, 8])
def test_stripes_virtual_ranks(feves, g):
    """P11 on the GPU: me_set_rows stripes (as the ranks of a G-GPU run would) == full frame."""
    W, H, S, n_rf = 320, 200, 32, 2     # 13 MB rows, ragged bottom
    cf, rfs = _frames("tex", W, H, n_rf, 42)
    me = feves.MotionEstimator(W, H, S, n_rf)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (fm, fs), (fq, fqs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    base, extra = divmod(me.mb_rows, g)
    r0 = 0
    for i in range(g):
        r1 = r0 + base + (1 if i < extra else 0)
        me.set_rows(r0, r1)
        sfs_s = [me.new_sf() for _ in trfs]
        (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs_s, n_int=n_rf, out_me=me.new_mvs())
        assert torch.equal(m, fm[r0:r1]) and torch.equal(s, fs[r0:r1])
        assert torch.equal(q, fq[r0:r1]) and torch.equal(qs, fqs[r0:r1])
        r0 = r1
    me.close()


def test_stream_push_ippp(feves, orc):
    """IPPP stream: frame t is searched over frames t-1..t-min(t,n_rf) (RF ramp)."""
    W, H, S, n_rf = 80, 48, 16, 3
    frames = [gen_tex(W, H, t, 61) for t in range(6)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    n = me.mb_rows * me.mb_cols
    for t, f in enumerate(frames):
        qm, qs = me.new_mvs()
        qm.fill_(-1)
        qm, qs, used = me.stream_push(_dev(f), out=(qm, qs))
        torch.cuda.synchronize()
        assert used == min(t, n_rf)
        if used == 0:
            continue
        rfs = [frames[t - 1 - k] for k in range(used)]
        o_mvs, _ = orc.me(f, rfs, S)
        o_q, o_s = orc.sme(f, rfs, o_mvs)
        gq = qm.cpu().numpy().reshape(n, n_rf, 41, 2)
        gs = qs.cpu().numpy().reshape(n, n_rf, 41)
        np.testing.assert_array_equal(gq[:, :used], o_q)
        np.testing.assert_array_equal(gs[:, :used], o_s)
        assert (gq[:, used:] == -1).all()            # untouched
    me.close()


def test_stream_push_host_buffers(feves, orc):
    W, H, S, n_rf = 64, 48, 8, 2
    frames = [gen_noise(W, H, t, 3) for t in range(4)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    n = me.mb_rows * me.mb_cols
    out = (torch.empty(me.mv_shape() + (2,), dtype=torch.int16).pin_memory(),
           torch.empty(me.mv_shape(), dtype=torch.uint16).pin_memory())
    for t, f in enumerate(frames):
        qm, qs, used = me.stream_push(torch.from_numpy(f).pin_memory(), out=out)
        me.sync()
    rfs = [frames[2], frames[1]]
    o_mvs, _ = orc.me(frames[3], rfs, S)
    o_q, o_s = orc.sme(frames[3], rfs, o_mvs)
    np.testing.assert_array_equal(qm.numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.numpy().reshape(n, n_rf, 41), o_s)
    me.close()


@pytest.mark.parametrize("graph", [0, 1])
def test_stream_host_pipeline_many_frames(feves, orc, graph):
    """host pushes back to back (uploads/downloads overlap compute on copy streams), with
    ME_OPT_GRAPH off and on (host pushes are never captured): every frame's host outputs,
    captured into its own pinned buffer, match the oracle"""
    W, H, S, n_rf = 64, 48, 8, 2
    frames = [gen_tex(W, H, t, 23) for t in range(11)]
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_option(me.OPT_GRAPH, graph)
    n = me.mb_rows * me.mb_cols
    outs = []
    for f in frames:
        o = (torch.empty(me.mv_shape() + (2,), dtype=torch.int16).pin_memory(),
             torch.empty(me.mv_shape(), dtype=torch.uint16).pin_memory())
        me.stream_push(torch.from_numpy(f).pin_memory(), out=o)
        outs.append(o)
    me.sync()
    for t in range(n_rf, len(frames)):
        rfs = [frames[t - 1 - k] for k in range(n_rf)]
        o_mvs, _ = orc.me(frames[t], rfs, S)
        o_q, o_s = orc.sme(frames[t], rfs, o_mvs)
        np.testing.assert_array_equal(outs[t][0].numpy().reshape(n, n_rf, 41, 2), o_q)
        np.testing.assert_array_equal(outs[t][1].numpy().reshape(n, n_rf, 41), o_s)
    me.close()


@pytest.mark.parametrize("lam,S", [(4, 16), (25, 32), (200, 8), (9, 128)])
def test_rate_term_me_sme_and_mode_decision(feves, orc, lam, S):
    """f4 (G18) and f2 (O4) on the GPU path vs the oracle, bit-exact"""
    W, H, n_rf = 80, 48, 2
    cf, rfs = _frames("tex", W, H, n_rf, 3 + lam)
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_lambda(lam)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    modes = me.mode_decision(q, qs)
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, o_s = orc.me(cf, rfs, S, lam=lam)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, n_rf, 41, 2), o_m)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, n_rf, 41), o_s)
    o_q, o_qs = orc.sme(cf, rfs, o_m, lam=lam)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_qs)
    np.testing.assert_array_equal(modes.cpu().numpy().reshape(n, 10), orc.mode_decision(o_q, o_qs, lam))
    me.set_lambda(0)                                     # back to pure SAD: original results
    (m0, s0), _ = me.encode_frame(tcf, trfs, sfs, n_int=0, out_me=me.new_mvs())
    torch.cuda.synchronize()
    o_m0, o_s0 = orc.me(cf, rfs, S)
    np.testing.assert_array_equal(m0.cpu().numpy().reshape(n, n_rf, 41, 2), o_m0)
    me.close()


@pytest.mark.parametrize("lam,S,kind", [(0, 16, "tex"), (6, 32, "noise"), (0, 8, "flat")])
def test_sme_satd(feves, orc, lam, S, kind):
    """f4 (G20): Hadamard-SATD SME on the GPU == oracle (with and without the rate term)"""
    W, H, n_rf = 64, 48, 2
    cf, rfs = _frames(kind, W, H, n_rf, 77 + S)
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_sme_satd(True)
    if lam:
        me.set_lambda(lam)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, _ = orc.me(cf, rfs, S, lam=lam)
    o_q, o_qs = orc.sme(cf, rfs, o_m, lam=lam, satd=True)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, n_rf, 41, 2), o_m)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_qs)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    me.close()


@pytest.mark.parametrize("W,H,S,n_rf,kind,lam", [
    (64, 48, 16, 2, "tex", 0), (72, 52, 32, 1, "noise", 0), (40, 40, 128, 1, "noise", 0),
    (50, 30, 6, 1, "flat", 0), (80, 48, 64, 2, "tex", 0), (64, 48, 16, 2, "tex", 9)])
def test_sa_inclusive(feves, orc, W, H, S, n_rf, kind, lam):
    """f4 (G1 alternative reading): candidates [-S/2, +S/2]^2 on the GPU == oracle(sa_inclusive=True),
    then SME on those MVs; switching back restores the base reading's results"""
    cf, rfs = _frames(kind, W, H, n_rf, 500 + S + lam)
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_sa_inclusive(True)
    if lam:
        me.set_lambda(lam)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, o_s = orc.me(cf, rfs, S, sa_inclusive=True, lam=lam)
    np.testing.assert_array_equal(m.cpu().numpy().reshape(n, n_rf, 41, 2), o_m)
    np.testing.assert_array_equal(s.cpu().numpy().reshape(n, n_rf, 41), o_s)
    assert np.abs(o_m).max() <= S // 2
    o_q, o_qs = orc.sme(cf, rfs, o_m, lam=lam)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_qs)
    me.set_sa_inclusive(False)
    (m0, s0), _ = me.encode_frame(tcf, trfs, sfs, n_int=0, out_me=me.new_mvs())
    torch.cuda.synchronize()
    o_m0, o_s0 = orc.me(cf, rfs, S, lam=lam)
    np.testing.assert_array_equal(m0.cpu().numpy().reshape(n, n_rf, 41, 2), o_m0)
    np.testing.assert_array_equal(s0.cpu().numpy().reshape(n, n_rf, 41), o_s0)
    me.close()


@pytest.mark.parametrize("host", [False, True])
def test_stream_overlap_sme_equals_serial(feves, host):
    """ME_OPT_OVERLAP_SME (SME(t) co-runs with ME(t+1) on its own stream): every frame's
    outputs, each pushed into its own buffer, equal the serial stream's, bitwise; with a
    large frame so that the kernels really overlap, and the RF ramp included."""
    W, H, S, n_rf = 640, 360, 32, 4
    frames = [gen_tex(W, H, t, 71) for t in range(9)]

    def run(overlap):
        me = feves.MotionEstimator(W, H, S, n_rf)
        me.set_option(me.OPT_OVERLAP_SME, int(overlap))
        outs = []
        for f in frames:
            if host:
                o = (torch.full(me.mv_shape() + (2,), -7, dtype=torch.int16).pin_memory(),
                     torch.full(me.mv_shape(), 7, dtype=torch.uint16).pin_memory())
                src = torch.from_numpy(f).pin_memory()
            else:
                o = (torch.full(me.mv_shape() + (2,), -7, dtype=torch.int16, device="cuda"),
                     torch.full(me.mv_shape(), 7, dtype=torch.uint16, device="cuda"))
                src = _dev(f)
            _, _, used = me.stream_push(src, out=o)
            outs.append((o, used))
        me.sync()
        torch.cuda.synchronize()
        res = [(o[0].cpu().numpy(), o[1].cpu().numpy(), u) for o, u in outs]
        me.close()
        return res

    a, b = run(False), run(True)
    for (qa, sa, ua), (qb, sb, ub) in zip(a, b):
        assert ua == ub
        np.testing.assert_array_equal(qa, qb)
        np.testing.assert_array_equal(sa, sb)
    assert any(u == n_rf for _, _, u in a)


@pytest.mark.parametrize("n_rf,halo", [(2, False), (4, True)])
def test_stream_graph_replay_equals_oracle(feves, orc, n_rf, halo):
    """ME_OPT_GRAPH (SURVEY §8(d) one CUDA graph per frame): steady-state pushes are captured
    once per ring phase (period lcm(n_rf+2, n_rf, 2)) and REPLAYED; the frames come from 5
    distinct device tensors (the graph's copy node is re-pointed) into ONE output buffer, and
    a stripe change mid-stream re-captures.  Every frame's outputs == the oracle."""
    W, H, S = 80, 64, 16
    frames = [gen_tex(W, H, t, 83) for t in range(3 * (n_rf + 2) * n_rf + 4)]
    dev = [_dev(f) for f in frames[:5]]
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_option(me.OPT_GRAPH, 1)
    if halo:
        me.set_option(me.OPT_HALO_ONLY, 1)
        me.set_rows(1, 3)
    out = me.new_mvs()
    n_checked = 0
    for t, f in enumerate(frames):
        src = dev[t % 5]
        src.copy_(_dev(f))                               # torch stream == context stream: ordered
        if t == len(frames) - 3 and not halo:
            me.set_rows(1, 4)                            # re-capture with another stripe
            out = me.new_mvs()
        qm, qs, used = me.stream_push(src, out=out)
        if used < n_rf and t > n_rf:
            raise AssertionError("ramp")
        if t % 3 == 0 or t >= len(frames) - 4:           # oracle on a subset of the frames
            torch.cuda.synchronize()
            rfs = [frames[t - 1 - k] for k in range(used)]
            mbs = orc.all_mbs(W, H, me.row0, me.row1)
            if not used:
                continue
            o_m, _ = orc.me(f, rfs, S, mb_list=mbs)
            o_q, o_s = orc.sme(f, rfs, o_m, mb_list=mbs)
            n = len(mbs)
            np.testing.assert_array_equal(qm.cpu().numpy().reshape(n, n_rf, 41, 2)[:, :used], o_q, err_msg=str(t))
            np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41)[:, :used], o_s, err_msg=str(t))
            n_checked += 1
    assert n_checked >= 8
    me.close()


@pytest.mark.parametrize("lam,S,kind", [(0, 64, "tex"), (0, 32, "noise"), (7, 16, "flat"), (0, 128, "tex")])
def test_sme_staged_kernel_equals_oracle(feves, orc, lam, S, kind):
    """ME_OPT_SME_KERNEL = 1: the shared-memory staged SME (TMA-staged sub-pel footprint box per
    8-MB group; boxes beyond the region through the overflow list) == oracle, with and without
    the rate term, on frames wide enough for several groups and a ragged last group"""
    W, H, n_rf = 200, 72, 2                              # 13 MBs per row: groups of 8 + 5
    cf, rfs = _frames(kind, W, H, n_rf, 91 + S + lam)
    me = feves.MotionEstimator(W, H, S, n_rf)
    me.set_option(me.OPT_SME_KERNEL, 1)
    if lam:
        me.set_lambda(lam)
    tcf, trfs = _dev(cf), [_dev(r) for r in rfs]
    sfs = [me.new_sf() for _ in trfs]
    (m, s), (q, qs) = me.encode_frame(tcf, trfs, sfs, n_int=n_rf, out_me=me.new_mvs())
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    o_m, _ = orc.me(cf, rfs, S, lam=lam)
    o_q, o_qs = orc.sme(cf, rfs, o_m, lam=lam)
    np.testing.assert_array_equal(q.cpu().numpy().reshape(n, n_rf, 41, 2), o_q)
    np.testing.assert_array_equal(qs.cpu().numpy().reshape(n, n_rf, 41), o_qs)
    me.close()


@pytest.mark.parametrize("W,H,S", [(64, 48, 8), (72, 52, 16), (854, 40, 32), (330, 170, 64), (33, 17, 128)])
def test_int_kernels_equal_oracle(feves, orc, W, H, S):
    """both INT kernels (ME_OPT_INT_KERNEL 0: per-thread global loads, 1: shared-memory tiles)
    write every byte of the 16 planes == oracle, incl. ragged tiles and W % 4 != 0"""
    rf = gen_noise(W, H, 0, W * H + S)
    me = feves.MotionEstimator(W, H, S, 1)
    ref = orc.int_planes(rf, me.sf_pad, me.sf_pitch, me.sf_rows)
    for k in (0, 1):
        me.set_option(me.OPT_INT_KERNEL, k)
        sf = me.new_sf()
        sf.fill_(0x5A)
        me.interpolate(_dev(rf), out=sf)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(sf.cpu().numpy(), ref, err_msg=f"int_kernel={k}")
    me.close()
