"""GPU parity at BASELINE.json's full sizes, EVERY MB, through the path bench.py times.

SURVEY §8(c)/(d): "Parity: full on configs 1-4.  On config 5, ... every row adjacent to a
stripe boundary".  The workloads are the paper's 1080p/2160p IPPP sequences (P:258-P:260);
frames come from synth.ippp_sequence with bench.py's seeds (1000 + config index).  Every
frame of an IPPP stream of >= n_rf + 2 frames is pushed through me_stream_push -- with
PINNED HOST frames and HOST outputs (the e2e entry of the bench line) and with device
buffers (the `value` entry) -- and every MB of every frame (RF ramp included) is
compared with the CPU oracle (O1 ME + O3 SME over the frame's min(t, n_rf) RFs, G15),
bit-exact.  Config 4 (config 3 split into MB-row stripes) reuses config 3's
oracle results: every stripe of every 2/4/8-way split, pushed as its rank would (halo-only
copies), equals them.  The oracle costs ~8 s per RF per 1080p S64 frame on 16 cores.
"""
import numpy as np
import pytest
import torch

from synth import CONFIGS, ippp_sequence

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def feves():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    assert torch.cuda.is_available()
    return pkg


def _stripes(n, g):
    base, extra = divmod(n, g)
    out, r0 = [], 0
    for i in range(g):
        r1 = r0 + base + (1 if i < extra else 0)
        out.append((r0, r1))
        r0 = r1
    return out


def _oracle_frames(orc, frames, n_rf, S, mbs=None):
    """{t: (qmvs, qsads)} of the oracle for every frame t >= 1 of an IPPP sequence"""
    res = {}
    for t in range(1, len(frames)):
        rfs = [frames[t - 1 - k] for k in range(min(t, n_rf))]
        o_m, o_s = orc.me(frames[t], rfs, S, mb_list=mbs)
        o_q, o_qs = orc.sme(frames[t], rfs, o_m, mb_list=mbs)
        res[t] = (o_m, o_s, o_q, o_qs)
    return res


def _push_all(feves, cfg, frames, host, rows=None, halo_only=False, graph=False):
    """push every frame; returns [(qmvs, qsads, used)] as numpy, one output buffer per frame"""
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
    if graph:
        me.set_option(me.OPT_GRAPH, 1)
    if rows is not None:
        me.set_rows(*rows)
    if halo_only:
        me.set_option(me.OPT_HALO_ONLY, 1)
    outs = []
    for f in frames:
        if host:
            o = (torch.full(me.mv_shape() + (2,), -9, dtype=torch.int16).pin_memory(),
                 torch.full(me.mv_shape(), 9, dtype=torch.uint16).pin_memory())
            src = torch.from_numpy(f).pin_memory()
        else:
            o = (torch.full(me.mv_shape() + (2,), -9, dtype=torch.int16, device="cuda"),
                 torch.full(me.mv_shape(), 9, dtype=torch.uint16, device="cuda"))
            src = torch.from_numpy(f).cuda()
        _, _, used = me.stream_push(src, out=o)
        outs.append((o, used))
    me.sync()
    torch.cuda.synchronize()
    res = [(o[0].cpu().numpy(), o[1].cpu().numpy(), u) for o, u in outs]
    me.close()
    return res


def _compare(res, ref, n_rf, mb_slice=slice(None)):
    for t, (qm, qs, used) in enumerate(res):
        assert used == min(t, n_rf)
        if not used:
            continue
        n = qs.shape[0] * qs.shape[1]
        _, _, o_q, o_qs = ref[t]
        np.testing.assert_array_equal(qs.reshape(n, n_rf, 41)[:, :used], o_qs[mb_slice], err_msg=f"frame {t}")
        np.testing.assert_array_equal(qm.reshape(n, n_rf, 41, 2)[:, :used], o_q[mb_slice], err_msg=f"frame {t}")
        assert (qm.reshape(n, n_rf, 41, 2)[:, used:] == -9).all()        # RF slots not searched: untouched


@pytest.fixture(scope="module")
def config3(orc):
    cfg = CONFIGS["1080p_sa64_4rf"]
    frames = ippp_sequence(cfg.width, cfg.height, cfg.n_rf + 2, 1000 + cfg.baseline_index)
    return cfg, frames, _oracle_frames(orc, frames, cfg.n_rf, cfg.sa_range)


@pytest.mark.parametrize("host,graph", [(True, False), (True, True), (False, False), (False, True)])
def test_config3_1080p_s64_4rf_stream_every_mb(feves, config3, host, graph):
    """BASELINE config 3 (the bench workload): 1080p, 4 RFs, SA 64x64, INT || ME -> SME through
    me_stream_push (host buffers = bench e2e, with ME_OPT_GRAPH set too -- it applies to device
    pushes only; device buffers, captured as CUDA graphs = bench value), 6 frames (RF ramp 1, 2, 3,
    4, 4), every MB of every frame == oracle."""
    cfg, frames, ref = config3
    _compare(_push_all(feves, cfg, frames, host, graph=graph), ref, cfg.n_rf)


@pytest.mark.parametrize("g", [2, 4, 8])
def test_config4_1080p_sharded_every_mb(feves, config3, g):
    """BASELINE config 4: config 3 MB-row sharded over g ranks (equidistant split); each
    rank's stripe pushed with halo-only copies (its stripe + SA halo rows), every
    MB of every stripe of every frame == oracle (the union covers the frame)."""
    cfg, frames, ref = config3
    mbc = -(-cfg.width // 16)
    for r0, r1 in _stripes(-(-cfg.height // 16), g):
        res = _push_all(feves, cfg, frames, host=(r0 == 0), rows=(r0, r1), halo_only=True)
        _compare(res, ref, cfg.n_rf, slice(r0 * mbc, r1 * mbc))


def test_config2_1080p_s32_stream_every_mb(feves, orc):
    """BASELINE config 2: 1080p, 1 RF, SA 32x32 integer FSBM; 3 frames through the host-buffer
    stream (every MB of frames 1 and 2, SME included) and me_estimate (ME MVs/SADs, every MB)."""
    cfg = CONFIGS["1080p_sa32"]
    frames = ippp_sequence(cfg.width, cfg.height, cfg.n_rf + 2, 1000 + cfg.baseline_index)
    ref = _oracle_frames(orc, frames, cfg.n_rf, cfg.sa_range)
    _compare(_push_all(feves, cfg, frames, host=True), ref, cfg.n_rf)
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
    mvs, sads = me.estimate(torch.from_numpy(frames[2]).cuda(), [torch.from_numpy(frames[1]).cuda()])
    torch.cuda.synchronize()
    n = me.mb_rows * me.mb_cols
    np.testing.assert_array_equal(sads.cpu().numpy().reshape(n, 1, 41), ref[2][1])
    np.testing.assert_array_equal(mvs.cpu().numpy().reshape(n, 1, 41, 2), ref[2][0])
    me.close()


def test_config5_2160p_s128_stripe_boundary_rows(feves, orc):
    """BASELINE config 5: 2160p, 4 RFs, SA 128x128, MB-row sharded over 8 ranks (17 x 7 + 16
    rows): each rank's stripe pushed as that rank would (halo-only copies), 5 frames; at the
    last frame (all 4 RFs) every MB of every row adjacent to a stripe boundary, plus the
    first and last rows of the frame, == oracle (ME on 16384 candidates per MB and RF)."""
    cfg = CONFIGS["2160p_sa128"]
    frames = ippp_sequence(cfg.width, cfg.height, cfg.n_rf + 1, 1000 + cfg.baseline_index)
    mbc, mbr = -(-cfg.width // 16), -(-cfg.height // 16)
    st = _stripes(mbr, 8)
    rows = sorted({0, mbr - 1} | {r for r0, r1 in st for r in (r0, r1 - 1)})
    mbs = np.array([r * mbc + c for r in rows for c in range(mbc)], np.int32)
    t = cfg.n_rf
    rfs = [frames[t - 1 - k] for k in range(cfg.n_rf)]
    o_m, o_s = orc.me(frames[t], rfs, cfg.sa_range, mb_list=mbs)
    o_q, o_qs = orc.sme(frames[t], rfs, o_m, mb_list=mbs)
    for r0, r1 in st:
        res = _push_all(feves, cfg, frames, host=False, rows=(r0, r1), halo_only=True)
        qm, qs, used = res[t]
        assert used == cfg.n_rf
        for r in (r0, r1 - 1):
            k = rows.index(r)
            sl = slice(k * mbc, (k + 1) * mbc)
            np.testing.assert_array_equal(qs[r - r0], o_qs[sl].reshape(mbc, cfg.n_rf, 41), err_msg=f"row {r}")
            np.testing.assert_array_equal(qm[r - r0], o_q[sl].reshape(mbc, cfg.n_rf, 41, 2), err_msg=f"row {r}")
