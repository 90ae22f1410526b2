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
