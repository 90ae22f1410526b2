"""Multi-process sharding plumbing on CPU (gloo, world_size 2 and 3).

The compute backend here is an oracle-backed stand-in (tests may call the
oracle; the product path never does).  It checks the broadcast-in /
stripe-push / gather-out logic of paper_conf_icpp_ilicmrs14_b200.shard: the
assembled outputs on rank 0 equal the full-frame oracle, frame after frame,
including the RF ramp.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from synth import gen_tex

W, H, S, N_RF, N_FRAMES = 48, 72, 8, 2, 4     # 5 MB rows (ragged bottom)


class OracleStripeBackend:
    """Stand-in for MotionEstimator.stream_push on one stripe, computed by the oracle."""

    def __init__(self, r0, r1):
        import oracle
        self.orc = oracle
        self.row0, self.row1 = r0, r1
        self.mb_cols, self.mb_rows = -(-W // 16), -(-H // 16)
        self.ring = []

    def mv_shape(self):
        return (self.row1 - self.row0, self.mb_cols, N_RF, 41)

    def stream_push(self, frame):
        from paper_conf_icpp_ilicmrs14_b200.shard import halo_rows
        f = frame.numpy().copy()
        # a rank only trusts its stripe + halo rows: corrupt the rest to prove it
        lo, hi = halo_rows(self.row0, self.row1, S, H)
        f[:lo] = 255
        f[hi:] = 0
        t = len(self.ring)
        self.ring.append(f)
        n_ref = min(t, N_RF)
        qm = torch.zeros(self.mv_shape() + (2,), dtype=torch.int16)
        qs = torch.zeros(self.mv_shape(), dtype=torch.uint16)
        if n_ref:
            rfs = [self.ring[t - 1 - k] for k in range(n_ref)]
            mbs = np.arange(self.row0 * self.mb_cols, self.row1 * self.mb_cols, dtype=np.int32)
            mv, _ = self.orc.me(f, rfs, S, mb_list=mbs)
            q, s = self.orc.sme(f, rfs, mv, mb_list=mbs)
            qm[:, :, :n_ref] = torch.from_numpy(q.reshape(self.row1 - self.row0, self.mb_cols, n_ref, 41, 2))
            qs[:, :, :n_ref] = torch.from_numpy(s.reshape(self.row1 - self.row0, self.mb_cols, n_ref, 41))
        return qm, qs, n_ref


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_ilicmrs14_b200.shard import ShardedStream, stripes
        r0, r1 = stripes(-(-H // 16), world)[rank]
        ss = ShardedStream(OracleStripeBackend(r0, r1))
        frames = [gen_tex(W, H, t, 5) for t in range(N_FRAMES)]
        buf = torch.zeros(H, W, dtype=torch.uint8)
        outs = []
        for t in range(N_FRAMES):
            src = torch.from_numpy(frames[t]) if rank == 0 else buf
            r = ss.push(src, buf)
            if rank == 0:
                outs.append((r[0].numpy(), r[1].numpy(), r[2]))
        if rank == 0:
            q.put(outs)
    finally:
        dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_stream_equals_full_frame(orc, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    frames = [gen_tex(W, H, t, 5) for t in range(N_FRAMES)]
    n = (-(-W // 16)) * (-(-H // 16))
    for t, (qm, qs, n_ref) in enumerate(outs):
        assert n_ref == min(t, N_RF)
        if n_ref == 0:
            continue
        rfs = [frames[t - 1 - k] for k in range(n_ref)]
        mv, _ = orc.me(frames[t], rfs, S)
        oq, os_ = orc.sme(frames[t], rfs, mv)
        np.testing.assert_array_equal(qm.reshape(n, N_RF, 41, 2)[:, :n_ref], oq)
        np.testing.assert_array_equal(qs.reshape(n, N_RF, 41)[:, :n_ref], os_)


def test_stripes_and_halo():
    from paper_conf_icpp_ilicmrs14_b200.shard import halo_rows, stripes
    assert stripes(68, 8) == [(0, 9), (9, 18), (18, 27), (27, 36), (36, 44), (44, 52), (52, 60), (60, 68)]
    assert [b - a for a, b in stripes(135, 8)] == [17] * 7 + [16]
    assert stripes(68, 2) == [(0, 34), (34, 68)]
    assert halo_rows(0, 9, 64, 1080) == (0, 144 + 35)
    assert halo_rows(60, 68, 64, 1080) == (960 - 35, 1080)


# ------------------------------------------------------------- f3: adaptive split --

def test_split_rows_properties():
    from paper_conf_icpp_ilicmrs14_b200.shard import split_rows, stripes
    assert split_rows(68, [1] * 8) == stripes(68, 8)
    for n, w in [(68, [1, 2]), (135, [3, 1, 1, 5, 2, 2, 1, 1]), (5, [100, 1, 1]), (8, [1] * 8)]:
        st = split_rows(n, w)
        assert st[0][0] == 0 and st[-1][1] == n
        assert all(a < b for a, b in st) and all(st[i][1] == st[i + 1][0] for i in range(len(st) - 1))
    st = split_rows(90, [2, 1])
    assert [b - a for a, b in st] == [60, 30]


def test_adaptive_split_converges_to_inverse_cost():
    from paper_conf_icpp_ilicmrs14_b200.shard import AdaptiveSplit
    cost = [1.0, 3.0, 1.0]                    # time per MB row on each device
    a = AdaptiveSplit(60, 3, smoothing=0.0)
    for _ in range(3):
        st = a.stripes()
        a.update([cost[i] * (b - e) for i, (e, b) in enumerate(st)])
    rows = [b - e for e, b in a.stripes()]
    assert rows == [26, 8, 26] or rows == [26, 9, 25] or rows == [25, 9, 26], rows   # 60 * (1, 1/3, 1) / (7/3)
    assert max(c * m for c, m in zip(cost, rows)) < max(c * 20 for c in cost)          # beats equidistant


class SlowRankTimer:
    """stripe 'time' = rows x per-rank cost (rank 1 is 3x slower): a deterministic stand-in
    for the CUDA-event timer, so the test is about the control loop, not the host clock."""

    def __init__(self, rank, backend):
        self.rank, self.be = rank, backend

    def __call__(self, fn):
        out = fn()
        return out, (3.0 if self.rank == 1 else 1.0) * (self.be.row1 - self.be.row0)


def _adaptive_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_ilicmrs14_b200.shard import ShardedStream, stripes
        mbr = -(-H2 // 16)
        be = OracleStripeBackend2(*stripes(mbr, world)[rank])
        ss = ShardedStream(be, adaptive=True, timer=SlowRankTimer(rank, be))
        frames = [gen_tex(W2, H2, t, 9) for t in range(N2)]
        buf = torch.zeros(H2, W2, dtype=torch.uint8)
        outs = []
        for t in range(N2):
            r = ss.push(torch.from_numpy(frames[t]) if rank == 0 else buf, buf)
            if rank == 0:
                outs.append((r[0].numpy(), r[1].numpy(), r[2]))
        if rank == 0:
            q.put((outs, ss.history))
    finally:
        dist.destroy_process_group()


W2, H2, N2 = 32, 128, 5          # 8 MB rows


class OracleStripeBackend2(OracleStripeBackend):
    """as OracleStripeBackend but on the W2 x H2 frames and re-splittable (set_rows)"""

    def __init__(self, r0, r1):
        super().__init__(r0, r1)
        self.mb_cols, self.mb_rows = -(-W2 // 16), -(-H2 // 16)

    def set_rows(self, r0, r1):
        self.row0, self.row1 = r0, r1

    def stream_push(self, frame):
        from paper_conf_icpp_ilicmrs14_b200.shard import halo_rows
        f = frame.numpy().copy()
        t = len(self.ring)
        self.ring.append(f)                     # whole frames (as the CUDA ring)
        n_ref = min(t, N_RF)
        qm = torch.zeros(self.mv_shape() + (2,), dtype=torch.int16)
        qs = torch.zeros(self.mv_shape(), dtype=torch.uint16)
        if n_ref:
            lo, hi = halo_rows(self.row0, self.row1, S, H2)
            def view(g):                         # only stripe + halo rows are trusted
                g = g.copy(); g[:lo] = 7; g[hi:] = 250
                return g
            rfs = [view(self.ring[t - 1 - k]) for k in range(n_ref)]
            mbs = np.arange(self.row0 * self.mb_cols, self.row1 * self.mb_cols, dtype=np.int32)
            mv, _ = self.orc.me(view(f), rfs, S, mb_list=mbs)
            q, s = self.orc.sme(view(f), rfs, mv, mb_list=mbs)
            rows = self.row1 - self.row0
            qm[:, :, :n_ref] = torch.from_numpy(q.reshape(rows, self.mb_cols, n_ref, 41, 2))
            qs[:, :, :n_ref] = torch.from_numpy(s.reshape(rows, self.mb_cols, n_ref, 41))
        return qm, qs, n_ref


def test_adaptive_sharded_stream_moves_rows_and_stays_exact(orc):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_adaptive_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs, history = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert history[0] == [(0, 4), (4, 8)]                  # equidistant first frame
    assert history[-1][0][1] - history[-1][0][0] == 6      # rank 1 is 3x slower -> 6 / 2 rows
    frames = [gen_tex(W2, H2, t, 9) for t in range(N2)]
    n = (-(-W2 // 16)) * (-(-H2 // 16))
    for t, (qm, qs, n_ref) in enumerate(outs):
        if n_ref == 0:
            continue
        rfs = [frames[t - 1 - k] for k in range(n_ref)]
        mv, _ = orc.me(frames[t], rfs, S)
        oq, os_ = orc.sme(frames[t], rfs, mv)
        np.testing.assert_array_equal(qm.reshape(n, N_RF, 41, 2)[:, :n_ref], oq)
        np.testing.assert_array_equal(qs.reshape(n, N_RF, 41)[:, :n_ref], os_)


def test_adaptive_split_with_a_lagged_split():
    """AdaptiveSplit.update(times, split=...) charges the times to the split that produced them
    (PeerStream adapts with a lag of two frames, by when the split may already have moved):
    K_i = t_i / m_i per row, next m_i proportional to 1 / K_i (eq. (1))."""
    from paper_conf_icpp_ilicmrs14_b200.shard import AdaptiveSplit
    a = AdaptiveSplit(8, 2, smoothing=0.0)
    assert a.stripes() == [(0, 4), (4, 8)]
    old = a.stripes()
    a.update([4.0, 4.0], split=[(0, 2), (2, 8)])        # 2 rows in 4 s vs 6 rows in 4 s: K = 2, 2/3
    assert a.stripes() == [(0, 2), (2, 8)]
    a.update([1.0, 3.0], split=old)                     # K = 1/4, 3/4 -> 3:1
    assert a.stripes() == [(0, 6), (6, 8)]
