"""MB-row sharding across GPUs (one process per GPU, torch.distributed).

Paper: the frame's N MB rows are split among devices, m_i rows each with
sum m_i = N (eq. (1)); the first frame uses an equidistant
split.  On B200 every device is the same, so the split stays
equidistant (rank g gets floor(N/G) rows, +1 for g < N mod G), and the
paper's host-staged PCIe copies become NCCL collectives over
NVLink/NVSwitch:
  in   rank 0 broadcasts each new frame (it becomes the CF now and an RF for
       the next n_rf frames); every rank keeps its own RF/SF ring in its
       libfeves_me context, so older RFs are never re-sent;
  out  the stripe outputs (quarter-pel MVs + SADs) are gathered to rank 0.
Exactness: MB row r depends only on CF rows [16r, 16r+15] and RF rows
[16r-R-3, 16r+15+R+3] (pinned by tests/test_oracle_shard.py and
the GPU virtual-rank test), so the assembled result equals the 1-GPU result.

The compute backend is any object with ``row0, row1, mv_shape()`` and
``stream_push(frame) -> (qmvs, qsads, n_ref)`` -- a ``MotionEstimator`` on the
GPU path.  This module does argument plumbing only; it never computes.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def stripes(n_rows: int, g: int):
    """Equidistant contiguous MB-row split: list of (r0, r1)."""
    base, extra = divmod(n_rows, g)
    out, r0 = [], 0
    for i in range(g):
        r1 = r0 + base + (1 if i < extra else 0)
        out.append((r0, r1))
        r0 = r1
    return out


def split_rows(n_rows: int, weights):
    """Contiguous stripes with sizes proportional to ``weights`` (largest-remainder
    rounding, at least one row each): the m_i of eq. (1), sum m_i = N."""
    g = len(weights)
    tot = float(sum(weights))
    raw = [n_rows * w / tot for w in weights]
    m = [max(1, int(r)) for r in raw]
    while sum(m) > n_rows:                      # min-1 clamps can overshoot
        i = max((k for k in range(g) if m[k] > 1), key=lambda k: m[k] - raw[k])
        m[i] -= 1
    rem = sorted(range(g), key=lambda k: raw[k] - m[k], reverse=True)
    i = 0
    while sum(m) < n_rows:
        m[rem[i % g]] += 1
        i += 1
    out, r0 = [], 0
    for k in range(g):
        out.append((r0, r0 + m[k]))
        r0 += m[k]
    return out


class AdaptiveSplit:
    """Adaptive MB-row distribution: the paper's Framework Control
    (Alg. 1) on identical GPUs.  Frame 1 is split equidistantly; after
    each frame the Performance Characterization K_i = (time of device i) / (rows of
    device i) ("processing time per MB row") is updated, and the next split
    minimises max_i K_i m_i subject to sum m_i = N -- the optimum of Alg. 2's LP when
    only the ME/INT/SME rows are distributed -- i.e. m_i proportional to 1/K_i.
    ``smoothing`` is an exponential average of K (absorbs timer noise; a real change
    is tracked within a few frames)."""

    def __init__(self, n_rows: int, world: int, smoothing: float = 0.5):
        self.n_rows, self.world, self.alpha = n_rows, world, smoothing
        self.cur = stripes(n_rows, world)
        self.K = None

    def stripes(self):
        return list(self.cur)

    def update(self, times, split=None):
        """times[i] = device i's time for a frame computed with ``split`` (default: the current one)"""
        rows = [r1 - r0 for r0, r1 in (self.cur if split is None else split)]
        k_now = [max(t, 1e-9) / max(m, 1) for t, m in zip(times, rows)]
        self.K = k_now if self.K is None else [self.alpha * a + (1 - self.alpha) * b
                                               for a, b in zip(self.K, k_now)]
        self.cur = split_rows(self.n_rows, [1.0 / k for k in self.K])
        return self.stripes()


def halo_rows(r0: int, r1: int, sa_range: int, height: int):
    """Frame rows a stripe [r0, r1) reads: [16 r0 - R - 3, 16 r1 + R + 3) clamped."""
    R = sa_range // 2
    return max(0, 16 * r0 - R - 3), min(height, 16 * r1 + R + 3)


def cuda_event_timer(fn):
    """(fn(), seconds) measured with CUDA events on the current stream: the per-device
    execution time the Performance Characterization uses."""
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    out = fn()
    b.record()
    b.synchronize()
    return out, a.elapsed_time(b) / 1e3


class ShardedStream:
    """IPPP stream over G ranks: broadcast in, per-rank stripe push, gather out.

    With ``adaptive=True`` the stripes are re-split after every frame from the per-rank
    stripe times (AdaptiveSplit); results do not depend on the split
    (pin P11), the library recomputes the SF rows a new stripe needs."""

    def __init__(self, backend, group=None, src: int = 0, adaptive: bool = False, timer=None):
        self.be = backend
        self.group = group
        self.src = src
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.split = AdaptiveSplit(backend.mb_rows, self.world) if adaptive else None
        self.timer = timer or cuda_event_timer  # callable(fn) -> (result, seconds) for the stripe work
        self.history = []                       # stripes used per frame (adaptive mode)
        self._apply(self.split.stripes() if adaptive else stripes(backend.mb_rows, self.world))

    def _apply(self, st):
        self.cur = st
        r0, r1 = st[self.rank]
        if (getattr(self.be, "row0", None), getattr(self.be, "row1", None)) != (r0, r1):
            self.be.set_rows(r0, r1)
        self.max_rows = max(b - a for a, b in st)

    def _host_staged(self, t):
        # gloo has no CUDA gather: stage through the host (only used to smoke-test the
        # multi-rank path on a single GPU; NCCL moves device buffers directly)
        return dist.get_backend(self.group) == "gloo" and t.is_cuda

    def push(self, frame, frame_buf):
        """frame: this step's frame on rank ``src`` (any device tensor, ignored elsewhere);
        frame_buf: a same-shape buffer on every rank that receives it.
        Returns (qmvs, qsads, n_ref) for the WHOLE frame on rank src, None elsewhere."""
        if self.rank == self.src:
            if frame.data_ptr() != frame_buf.data_ptr():
                frame_buf.copy_(frame)
        if self._host_staged(frame_buf):
            h = frame_buf.cpu()
            dist.broadcast(h, self.src, group=self.group)
            frame_buf.copy_(h)
        else:
            dist.broadcast(frame_buf, self.src, group=self.group)
        if self.split is None:
            qm, qs, n_ref = self.be.stream_push(frame_buf)
            return self._gather(qm, qs, n_ref)
        (qm, qs, n_ref), secs = self.timer(lambda: self.be.stream_push(frame_buf))
        out = self._gather(qm, qs, n_ref)
        tdev = torch.device("cpu") if (dist.get_backend(self.group) == "gloo") else frame_buf.device
        times = [torch.zeros(1, dtype=torch.float64, device=tdev) for _ in range(self.world)]
        dist.all_gather(times, torch.tensor([secs], dtype=torch.float64, device=tdev), group=self.group)
        self.history.append(self.cur)
        self._apply(self.split.update([float(x) for x in times]))
        return out

    def _gather(self, qm, qs, n_ref):
        pad_m = qm.new_zeros((self.max_rows,) + tuple(qm.shape[1:]))
        pad_s = qs.new_zeros((self.max_rows,) + tuple(qs.shape[1:]))
        pad_m[: qm.shape[0]].copy_(qm)
        pad_s[: qs.shape[0]].copy_(qs)
        # one collective for both fields: view the int16/uint16 payloads as bytes
        payload = torch.cat([pad_m.view(torch.uint8).reshape(-1), pad_s.view(torch.uint8).reshape(-1)])
        dev = payload.device
        if self._host_staged(payload):
            payload = payload.cpu()
        if self.rank == self.src:
            bufs = [torch.empty_like(payload) for _ in range(self.world)]
            dist.gather(payload, bufs, dst=self.src, group=self.group)
            parts_m, parts_s = [], []
            nm = pad_m.numel() * 2
            for (r0, r1), b in zip(self.cur, bufs):
                m = b[:nm].view(torch.int16).reshape(pad_m.shape)[: r1 - r0]
                s = b[nm:].view(torch.uint16).reshape(pad_s.shape)[: r1 - r0]
                parts_m.append(m)
                parts_s.append(s)
            return torch.cat(parts_m).to(dev), torch.cat(parts_s).to(dev), n_ref
        dist.gather(payload, None, dst=self.src, group=self.group)
        return None


class PeerStream:
    """IPPP stream over G ranks with the exchange done in peer memory and ordered by
    stream-ordered flags ("Option to fuse the collective"; BJ north_star
    "reference-frame rows plus an SA-radius halo via ... P2P over NVLink"; P:51 / P:89: the
    transfers overlap the computation).  No collective and no host synchronisation per frame.

    Rank ``src`` owns two frame slots, two full-frame output buffers and a done-flag word per
    rank; every rank owns two ready-flag words.  All are exported (``me_ipc_export``) and
    mapped by the others (``me_ipc_open``).  Flags are only ever WAITED on locally and
    WRITTEN remotely (``me_stream_wait_value`` / ``me_stream_write_value``).  Per frame t:
      rank src, publish stream:  wait for the start of its push t-1 (so everything up to the
          consumer of frame t-2 and the waits for its done flags have run), copy frame t into
          slot t mod 2, write ready[t mod 2] = t+1 into every rank's flag words;
      every rank, its stream:    ``me_stream_push_flags``: the copy-in stream waits for its own
          ready[t mod 2] >= t+1, pulls ONLY its stripe + halo rows from rank src's slot
          (``ME_OPT_HALO_ONLY``, copy engine over NVLink) -- overlapping its compute of frame
          t-1 --, runs INT || ME -> SME with the SME stores going straight into its stripe's rows
          of rank src's output buffer t mod 2, then writes done[rank] = t+1 into rank src's
          memory;
      rank src, its stream:      waits for done[r] >= t+1 of every rank.
    Slot / buffer reuse: slot and output buffer t mod 2 are rewritten at frame t+2, whose
    ready flag is written only after rank src passed the done-waits of frame t and whatever its
    caller enqueued after push t (e.g. the D2H of frame t's outputs).  The tensors returned on
    rank src are complete in its stream order and stay valid until push t+2.  Results equal
    the single-GPU stream bitwise (pin P11).  ``stripe_ms()`` gives each push's device time on
    this rank (CUDA events).

    Split: equidistant, or with ``adaptive=True`` the paper's iterative phase (Alg. 1
    l.7-11) through ``AdaptiveSplit``: at push t every rank reads its own
    device time of frame t - ``lag`` (an event pair two frames old, so no stall on the frame in
    flight), the times are all-gathered over a CPU (gloo) group, and every rank applies the same
    new split to frame t.  Ranks then pull whole frames (no halo-only copies: a grown stripe needs
    rows a halo-only ring frame would lack); the library refreshes the SF rows a moved stripe
    reads.  ``timer(rank, rows, seconds) -> seconds`` may replace the measured time (tests)."""

    def __init__(self, me, group=None, src: int = 0, adaptive: bool = False, lag: int = 2, timer=None):
        import paper_conf_icpp_ilicmrs14_b200 as F
        self.F = F
        self.me, self.group, self.src = me, group, src
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.split = AdaptiveSplit(me.mb_rows, self.world) if adaptive else None
        self.lag, self.timer = lag, timer
        self.ctrl = dist.new_group(backend="gloo") if adaptive else None   # CPU control plane
        self.cur = stripes(me.mb_rows, self.world)
        self.history = []                                                    # split used per frame
        r0, r1 = self.cur[self.rank]
        me.set_rows(r0, r1)
        me.set_option(me.OPT_HALO_ONLY, 0 if adaptive else 1)
        dev = me.device
        H, W = me.height, me.width
        shape = (me.mb_rows, me.mb_cols, me.n_rf, 41)
        self.row_bytes = (me.mb_cols * me.n_rf * 41 * 4, me.mb_cols * me.n_rf * 41 * 2)
        self.ready = torch.zeros(2, dtype=torch.int32, device=dev)              # mine: waited on locally
        mine = [me.ipc_export(self.ready) + (8,)]
        if self.rank == src:
            self.frames = [torch.empty((H, W), dtype=torch.uint8, device=dev) for _ in range(2)]
            self.qm = [torch.empty(shape + (2,), dtype=torch.int16, device=dev) for _ in range(2)]
            self.qs = [torch.empty(shape, dtype=torch.uint16, device=dev) for _ in range(2)]
            self.done = torch.zeros(self.world, dtype=torch.int32, device=dev)
            bufs = self.frames + self.qm + self.qs + [self.done]
            mine += [me.ipc_export(b) + (b.numel() * b.element_size(),) for b in bufs]
        allx = [None] * self.world
        dist.all_gather_object(allx, mine, group=group)
        self.opened = []
        self.t = 0
        self.times = []
        err = None
        try:                                          # mapping + a stream-memory-operation probe
            self._map(allx, bufs if self.rank == src else None, dev)
        except Exception as e:                        # noqa: BLE001 -- reported collectively below
            err = e
        ok = torch.tensor([0 if err else 1], dtype=torch.int32,
                          device=dev if dist.get_backend(group) == "nccl" else "cpu")
        dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
        if not int(ok.item()):                        # every rank raises: the caller can fall back
            for p in self.opened:
                try:
                    me.ipc_close(p)
                except Exception:                     # noqa: BLE001
                    pass
            self.opened = []
            raise F.FevesError(f"PeerStream unavailable: {err or 'a peer rank failed'}")
        dist.barrier(group=group)

    def _map(self, allx, bufs, dev):
        me, src = self.me, self.src

        def open_(h):
            p = me.ipc_open(*h)
            self.opened.append(p)
            return p
        if self.rank == src:
            ptrs = [b.data_ptr() for b in bufs]
            # every rank's ready words (own: local address)
            self.ready_ptrs = [self.ready.data_ptr() if r == src else open_(allx[r][0]) for r in range(self.world)]
            self.pub = torch.cuda.Stream(device=dev)
            self.ev_start = [torch.cuda.Event(), torch.cuda.Event()]
        else:
            ptrs = [open_(h) for h in allx[src][1:]]
        self.f_ptr, self.qm_ptr, self.qs_ptr = ptrs[0:2], ptrs[2:4], ptrs[4:6]
        self.done_ptr = ptrs[6]                                              # rank src's done words
        # probe: a stream write into rank src's memory and a stream wait on local memory (raises
        # if this platform does not support stream memory operations on peer-mapped memory)
        probe = torch.cuda.current_stream(dev)
        self.F.stream_write_value(probe, self.done_ptr + 4 * self.rank, 0)
        self.F.stream_wait_value(probe, self.ready.data_ptr(), 0)
        probe.synchronize()

    def push(self, frame, frame_buf=None):
        """frame: this step's frame on rank ``src`` (device or pinned host tensor [H, W]);
        ignored elsewhere.  Returns (qmvs, qsads, n_ref) of the WHOLE frame on rank src
        (complete in its stream order), None elsewhere."""
        F, t, b = self.F, self.t, self.t & 1
        cs = torch.cuda.current_stream(self.me.device)
        if self.rank == self.src:
            self.ev_start[b].record(cs)
            with torch.cuda.stream(self.pub):
                if t >= 1:
                    self.pub.wait_event(self.ev_start[b ^ 1])               # start of push t-1
                self.frames[b].copy_(frame.view(self.me.height, self.me.width), non_blocking=True)
                for p in self.ready_ptrs:
                    F.stream_write_value(self.pub, p + 4 * b, t + 1)
        if self.split is not None and t >= self.lag:                         # Alg. 1 iterative phase
            k = t - self.lag
            a, z = self.times[k]
            z.synchronize()                                                  # frame t - lag: normally done
            secs = a.elapsed_time(z) / 1e3
            r0k, r1k = self.history[k][self.rank]
            if self.timer is not None:
                secs = self.timer(self.rank, r1k - r0k, secs)
            allt = [torch.zeros(1, dtype=torch.float64) for _ in range(self.world)]
            dist.all_gather(allt, torch.tensor([secs], dtype=torch.float64), group=self.ctrl)
            self.cur = self.split.update([float(x) for x in allt], split=self.history[k])
            self.me.set_rows(*self.cur[self.rank])
        self.history.append(list(self.cur))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(cs)
        r0 = self.cur[self.rank][0]
        n_ref = self.me.stream_push_flags(self.f_ptr[b], self.qm_ptr[b] + r0 * self.row_bytes[0],
                                          self.qs_ptr[b] + r0 * self.row_bytes[1],
                                          wait_flag=self.ready.data_ptr() + 4 * b, wait_value=t + 1,
                                          signal_flag=self.done_ptr + 4 * self.rank, signal_value=t + 1)
        e1.record(cs)
        self.times.append((e0, e1))
        self.t += 1
        if self.rank == self.src:
            for r in range(self.world):
                F.stream_wait_value(cs, self.done_ptr + 4 * r, t + 1)
            return self.qm[b], self.qs[b], n_ref
        return None

    def stripe_ms(self):
        """device time of each push on this rank (ms; CUDA events on its stream, P:87 / P:218)"""
        torch.cuda.synchronize(self.me.device)
        return [a.elapsed_time(b) for a, b in self.times]

    def close(self):
        """Unmap the peer buffers (collective: every rank keeps its exported memory alive until
        all have unmapped)."""
        self.me.sync()
        torch.cuda.synchronize(self.me.device)
        dist.barrier(group=self.group)
        for p in self.opened:
            self.me.ipc_close(p)
        self.opened = []
        dist.barrier(group=self.group)
