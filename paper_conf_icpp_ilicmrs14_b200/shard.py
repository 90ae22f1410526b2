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


def halo_rows(r0: int, r1: int, sa_range: int, height: int):
    """Frame rows a stripe [r0, r1) reads: [16 r0 - R - 3, 16 r1 + R + 3) clamped."""
    R = sa_range // 2
    return max(0, 16 * r0 - R - 3), min(height, 16 * r1 + R + 3)


class ShardedStream:
    """IPPP stream over G ranks: broadcast in, per-rank stripe push, gather out."""

    def __init__(self, backend, group=None, src: int = 0):
        self.be = backend
        self.group = group
        self.src = src
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.max_rows = max(r1 - r0 for r0, r1 in stripes(backend.mb_rows, self.world))

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
        qm, qs, n_ref = self.be.stream_push(frame_buf)
        return self._gather(qm, qs, n_ref)

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
            for (r0, r1), b in zip(stripes(self.be.mb_rows, self.world), bufs):
                m = b[:nm].view(torch.int16).reshape(pad_m.shape)[: r1 - r0]
                s = b[nm:].view(torch.uint16).reshape(pad_s.shape)[: r1 - r0]
                parts_m.append(m)
                parts_s.append(s)
            return torch.cat(parts_m).to(dev), torch.cat(parts_s).to(dev), n_ref
        dist.gather(payload, None, dst=self.src, group=self.group)
        return None
