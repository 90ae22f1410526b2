"""Multi-process MB-row sharding on the GPU path: 2-4 ranks (sharing cuda:0, gloo,
CPU-staged collectives) run ShardedStream / PeerStream over real MotionEstimator stripes;
rank 0's assembled quarter-pel MVs/SADs of EVERY frame must equal the CPU ORACLE (O1 + O3
over the frame's min(t, n_rf) RFs, G15), bitwise -- P11 on the CUDA path, through the same
code bench.py runs under torchrun, including the f3 adaptive re-split."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

W, H, S, N_RF, N_FRAMES = 160, 120, 32, 2, 5      # 8 MB rows, ragged bottom


def _oracle_matches(outs, frames_np):
    """rank 0's outputs of every frame vs the oracle (IPPP, RF k = frame t-1-k)"""
    import oracle
    n = ((H + 15) // 16) * ((W + 15) // 16)
    for t, (qm, qs, used) in enumerate(outs):
        if used != min(t, N_RF):
            return False
        if not used:
            continue
        rfs = [frames_np[t - 1 - k] for k in range(used)]
        o_m, _ = oracle.me(frames_np[t], rfs, S)
        o_q, o_s = oracle.sme(frames_np[t], rfs, o_m)
        if not (np.array_equal(qm.reshape(n, N_RF, 41, 2)[:, :used], o_q) and
                np.array_equal(qs.reshape(n, N_RF, 41)[:, :used], o_s)):
            return False
    return True


class _SlowRank1:
    def __init__(self, rank, be):
        self.rank, self.be = rank, be

    def __call__(self, fn):
        out = fn()
        torch.cuda.synchronize()
        return out, (3.0 if self.rank == 1 else 1.0) * (self.be.row1 - self.be.row0)


def _worker(rank, world, port, q, adaptive=False):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_ilicmrs14_b200 as F
        from paper_conf_icpp_ilicmrs14_b200.shard import ShardedStream, stripes
        from synth import gen_tex
        torch.cuda.set_device(0)
        me = F.MotionEstimator(W, H, S, N_RF)
        r0, r1 = stripes(me.mb_rows, world)[rank]
        me.set_rows(r0, r1)
        ss = ShardedStream(me, adaptive=adaptive, timer=_SlowRank1(rank, me) if adaptive else None)
        buf = torch.zeros(H, W, dtype=torch.uint8, device="cuda")
        frames_np = [gen_tex(W, H, t, 31) for t in range(N_FRAMES)]
        frames = [torch.from_numpy(f).cuda() for f in frames_np]
        outs = []
        for t in range(N_FRAMES):
            r = ss.push(frames[t], buf)
            if rank == 0:
                outs.append((r[0].cpu().numpy(), r[1].cpu().numpy(), r[2]))
        if rank == 0:
            ok = _oracle_matches(outs, frames_np)
            q.put((ok, ss.history))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("adaptive", [False, True])
def test_two_rank_sharded_stream_equals_oracle(adaptive):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, adaptive)) for r in range(2)]
    for p in procs:
        p.start()
    ok, history = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert ok
    if adaptive:                       # rank 1 reported 3x the time per row: rows moved to rank 0
        assert history[0] == [(0, 4), (4, 8)] and history[-1] == [(0, 6), (6, 8)]


def _slow_rank1_time(rank, rows, secs):
    return (3.0 if rank == 1 else 1.0) * rows


def _peer_worker(rank, world, port, q, host_frames, adaptive=False):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_ilicmrs14_b200 as F
        from paper_conf_icpp_ilicmrs14_b200.shard import PeerStream
        from synth import gen_tex
        torch.cuda.set_device(0)
        me = F.MotionEstimator(W, H, S, N_RF)
        ps = PeerStream(me, adaptive=adaptive, timer=_slow_rank1_time if adaptive else None)
        frames_np = [gen_tex(W, H, t, 37) for t in range(N_FRAMES)]
        frames = [torch.from_numpy(f) for f in frames_np]
        frames = [f.pin_memory() if host_frames else f.cuda() for f in frames]
        outs = []
        for t in range(N_FRAMES):
            r = ps.push(frames[t] if rank == 0 else None)
            if rank == 0:
                torch.cuda.synchronize()
                outs.append((r[0].cpu().numpy(), r[1].cpu().numpy(), r[2]))
        ps.close()
        if rank == 0:
            ok = _oracle_matches(outs, frames_np)
            q.put((ok, ps.history) if adaptive else ok)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,host_frames", [(2, False), (3, True), (4, False)])
def test_peer_stream_equals_oracle(world, host_frames):
    """PeerStream (SURVEY §8(e) fused exchange): frames pulled as stripe + halo rows from
    rank 0's IPC-exported slot, SME outputs stored straight into rank 0's IPC-exported
    buffer (no broadcast/gather) == the oracle on every frame, bitwise.  The ranks share
    cuda:0 here (same-device CUDA IPC); on the 8-GPU box the same stores cross NVLink."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    procs = [ctx.Process(target=_peer_worker, args=(r, world, port, q, host_frames)) for r in range(world)]
    for p in procs:
        p.start()
    ok = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert ok


def test_halo_only_push_refuses_missing_rows():
    """ME_OPT_HALO_ONLY copies only the stripe + halo rows; a later push whose stripe
    needs rows an older ring frame lacks must fail with ME_ESTATE, not read garbage."""
    import paper_conf_icpp_ilicmrs14_b200 as F
    from synth import gen_tex
    me = F.MotionEstimator(W, H, S, N_RF)
    me.set_rows(0, 2)
    me.set_option(me.OPT_HALO_ONLY, 1)
    frames = [torch.from_numpy(gen_tex(W, H, t, 41)).cuda() for t in range(3)]
    me.stream_push(frames[0])
    me.stream_push(frames[1])
    me.set_rows(6, 8)                   # rows 96..119 were never copied for frames 0, 1
    with pytest.raises(F.FevesError, match="state"):
        me.stream_push(frames[2])
    me.set_rows(0, 2)                   # the original stripe still works
    me.stream_push(frames[2])
    torch.cuda.synchronize()


def test_adaptive_peer_stream_equals_oracle():
    """f3 on the flag-ordered peer exchange: rank 1 reports 3x the time per MB row, so from frame
    lag = 2 on the split moves rows to rank 0 (Alg. 1's iterative phase; K_i per row);
    every frame's assembled output still equals the oracle (pin P11 + the library's SF refresh)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    procs = [ctx.Process(target=_peer_worker, args=(r, 2, port, q, False, True)) for r in range(2)]
    for p in procs:
        p.start()
    ok, history = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert ok
    assert history[0] == [(0, 4), (4, 8)] and history[1] == [(0, 4), (4, 8)]
    assert history[-1] == [(0, 6), (6, 8)]
