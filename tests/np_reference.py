"""Independent NumPy brute force for TINY inputs (pin P9 of DESIGN.md §4).

A second, differently-structured implementation of the definitions the C
oracle follows, used only to cross-check the oracle (never the CUDA path):
  * ME: vectorised over candidates on an edge-padded copy, argmin by
    lexicographic (SAD, rank) with the rank from the CLOSED FORM of G4 (the C
    oracle enumerates the spiral instead);
  * INT: whole-plane filtering of an edge-padded copy (the C oracle evaluates
    each sample independently);
  * SME: reads the NumPy planes (the C oracle calls its per-sample function).
Shares no code with oracle/ or with the CUDA library.
"""
from __future__ import annotations

import numpy as np

TAPS = np.array([1, -5, 20, 20, -5, 1], np.int64)


def rank_closed_form(dx, dy):
    dx = np.asarray(dx, np.int64)
    dy = np.asarray(dy, np.int64)
    l = np.maximum(np.abs(dx), np.abs(dy))
    base = (2 * l - 1) ** 2
    top = base + 2 * (dx + l - 1) + (dy > 0)
    side = base + 2 * (2 * l - 1) + 2 * (dy + l) + (dx > 0)
    r = np.where(np.abs(dy) > np.abs(dx), top, side)
    return np.where(l == 0, 0, r)


def partitions():
    """(ox, oy, w, h) in G7 order, built from the mode list (not index arithmetic)."""
    out = [(0, 0, 16, 16), (0, 0, 16, 8), (0, 8, 16, 8), (0, 0, 8, 16), (8, 0, 8, 16)]
    subs = [(0, 0), (8, 0), (0, 8), (8, 8)]
    out += [(sx, sy, 8, 8) for sx, sy in subs]
    out += [(sx, sy + 4 * k, 8, 4) for sx, sy in subs for k in range(2)]
    out += [(sx + 4 * k, sy, 4, 8) for sx, sy in subs for k in range(2)]
    out += [(sx + 4 * (k % 2), sy + 4 * (k // 2), 4, 4) for sx, sy in subs for k in range(4)]
    return out


def _edge(f, m):
    return np.pad(f.astype(np.int64), m, mode="edge")


def me(cf, rfs, S):
    H, W = cf.shape
    R = S // 2
    mbc, mbr = -(-W // 16), -(-H // 16)
    Wp, Hp = 16 * mbc, 16 * mbr
    cfp = _edge(cf, ((0, Hp - H), (0, Wp - W)))
    m = R + 1
    d = np.arange(-R, R)
    DX, DY = np.meshgrid(d, d)               # [dy_idx, dx_idx]
    rank = rank_closed_form(DX, DY).ravel()
    parts = partitions()
    mvs = np.zeros((mbr * mbc, len(rfs), 41, 2), np.int16)
    sads = np.zeros((mbr * mbc, len(rfs), 41), np.uint16)
    for r, rf in enumerate(rfs):
        rfp = _edge(rf, ((m, m + Hp - H), (m, m + Wp - W)))
        for mby in range(mbr):
            for mbx in range(mbc):
                for p, (ox, oy, w, h) in enumerate(parts):
                    x0, y0 = 16 * mbx + ox, 16 * mby + oy
                    blk = cfp[y0:y0 + h, x0:x0 + w]
                    cand = np.empty(S * S, np.int64)
                    for i, (dy, dx) in enumerate(zip(DY.ravel(), DX.ravel())):
                        ys, xs = y0 + dy + m, x0 + dx + m
                        cand[i] = np.abs(blk - rfp[ys:ys + h, xs:xs + w]).sum()
                    best = np.lexsort((rank, cand))[0]
                    o = mby * mbc + mbx
                    mvs[o, r, p] = (DX.ravel()[best], DY.ravel()[best])
                    sads[o, r, p] = cand[best]
    return mvs, sads


def _clip1(v):
    return np.clip(v, 0, 255)


def planes(rf, pad, pitch, rows):
    """16 phase planes [16, rows, pitch]; plane origin at integer (-pad, -pad)."""
    H, W = rf.shape
    mgn = pad + 24
    E = _edge(rf, mgn)                        # E[y+mgn, x+mgn] = ref(x, y) for the margin used

    def sub(dy, dx):                          # integer sample at plane grid + (dx, dy)
        y0, x0 = mgn - pad + dy, mgn - pad + dx
        return E[y0:y0 + rows, x0:x0 + pitch]

    def hraw(dy, dx):                         # b1-type horizontal raw at grid + (dx,dy)
        return sum(TAPS[k] * sub(dy, dx + k - 2) for k in range(6))

    def vraw(dy, dx):                         # h1-type vertical raw at grid + (dx,dy)
        return sum(TAPS[k] * sub(dy + k - 2, dx) for k in range(6))

    G, Hh, M = sub(0, 0), sub(0, 1), sub(1, 0)
    b = _clip1((hraw(0, 0) + 16) >> 5)
    h = _clip1((vraw(0, 0) + 16) >> 5)
    m = _clip1((vraw(0, 1) + 16) >> 5)
    s = _clip1((hraw(1, 0) + 16) >> 5)
    j1 = sum(TAPS[k] * vraw(0, k - 2) for k in range(6))   # horizontal over h1 (C does vertical over b1)
    j = _clip1((j1 + 512) >> 10)
    avg = lambda u, v: (u + v + 1) >> 1
    byname = {
        (0, 0): G, (1, 0): avg(G, b), (2, 0): b, (3, 0): avg(Hh, b),
        (0, 1): avg(G, h), (1, 1): avg(b, h), (2, 1): avg(b, j), (3, 1): avg(b, m),
        (0, 2): h, (1, 2): avg(h, j), (2, 2): j, (3, 2): avg(j, m),
        (0, 3): avg(M, h), (1, 3): avg(h, s), (2, 3): avg(j, s), (3, 3): avg(m, s),
    }
    out = np.zeros((16, rows, pitch), np.uint8)
    for (xf, yf), v in byname.items():
        out[4 * yf + xf] = v
    return out


RING1 = [(0, -1), (0, 1), (-1, -1), (1, -1), (-1, 0), (1, 0), (-1, 1), (1, 1)]


def sme(cf, rfs, mvs, S):
    H, W = cf.shape
    mbc, mbr = -(-W // 16), -(-H // 16)
    Wp, Hp = 16 * mbc, 16 * mbr
    R = S // 2
    pad = R + 8
    pitch, rows = Wp + 2 * pad, Hp + 2 * pad
    cfp = _edge(cf, ((0, Hp - H), (0, Wp - W)))
    parts = partitions()
    qmvs = np.zeros_like(mvs)
    sads = np.zeros(mvs.shape[:3], np.uint16)
    for r, rf in enumerate(rfs):
        P = planes(rf, pad, pitch, rows).astype(np.int64)
        for o in range(mbr * mbc):
            mby, mbx = divmod(o, mbc)
            for p, (ox, oy, w, h) in enumerate(parts):
                x0, y0 = 16 * mbx + ox, 16 * mby + oy
                blk = cfp[y0:y0 + h, x0:x0 + w]

                def sadq(vx, vy):
                    ph = 4 * (vy & 3) + (vx & 3)
                    yy, xx = y0 + (vy >> 2) + pad, x0 + (vx >> 2) + pad
                    return int(np.abs(blk - P[ph, yy:yy + h, xx:xx + w]).sum())

                c = (4 * int(mvs[o, r, p, 0]), 4 * int(mvs[o, r, p, 1]))
                best, bv = sadq(*c), c
                for sx, sy in RING1:
                    v = (c[0] + 2 * sx, c[1] + 2 * sy)
                    sv = sadq(*v)
                    if sv < best:
                        best, bv = sv, v
                c2 = bv
                for sx, sy in RING1:
                    v = (c2[0] + sx, c2[1] + sy)
                    sv = sadq(*v)
                    if sv < best:
                        best, bv = sv, v
                qmvs[o, r, p] = bv
                sads[o, r, p] = best
    return qmvs, sads


# ---------------------------------------------------- G18 rate term / O4 mode decision --

def se_bits(v):
    v = int(v)
    k = 2 * v - 1 if v > 0 else -2 * v
    return 2 * (k + 1).bit_length() - 1          # 2*floor(log2(k+1)) + 1


def me_rd(cf, rfs, S, lam):
    """brute force: lexicographic (SAD + lam*R(4mv), rank) minimum per partition"""
    H, W = cf.shape
    R = S // 2
    mbc, mbr = -(-W // 16), -(-H // 16)
    Wp, Hp = 16 * mbc, 16 * mbr
    cfp = _edge(cf, ((0, Hp - H), (0, Wp - W)))
    m = R + 1
    d = np.arange(-R, R)
    DX, DY = np.meshgrid(d, d)
    rank = rank_closed_form(DX, DY).ravel()
    rate = np.array([lam * (se_bits(4 * x) + se_bits(4 * y)) for x, y in zip(DX.ravel(), DY.ravel())])
    parts = partitions()
    mvs = np.zeros((mbr * mbc, len(rfs), 41, 2), np.int16)
    sads = np.zeros((mbr * mbc, len(rfs), 41), np.uint16)
    for r, rf in enumerate(rfs):
        rfp = _edge(rf, ((m, m + Hp - H), (m, m + Wp - W)))
        for o in range(mbr * mbc):
            mby, mbx = divmod(o, mbc)
            for p, (ox, oy, w, h) in enumerate(parts):
                x0, y0 = 16 * mbx + ox, 16 * mby + oy
                blk = cfp[y0:y0 + h, x0:x0 + w]
                cand = np.array([np.abs(blk - rfp[y0 + dy + m:y0 + dy + m + h, x0 + dx + m:x0 + dx + m + w]).sum()
                                 for dy, dx in zip(DY.ravel(), DX.ravel())])
                best = np.lexsort((rank, cand + rate))[0]
                mvs[o, r, p] = (DX.ravel()[best], DY.ravel()[best])
                sads[o, r, p] = cand[best]
    return mvs, sads


def mode_decision(qmvs, sads, lam):
    """enumerates every H.264 P-MB configuration (mb_type; per 8x8: sub_type, ref) explicitly"""
    import itertools
    n, n_rf = sads.shape[:2]
    J = sads.astype(np.int64) + lam * np.vectorize(se_bits)(qmvs[..., 0]) + lam * np.vectorize(se_bits)(qmvs[..., 1])
    sub_parts = {0: lambda s: [5 + s], 1: lambda s: [9 + 2 * s, 10 + 2 * s],
                 2: lambda s: [17 + 2 * s, 18 + 2 * s], 3: lambda s: [25 + 4 * s + k for k in range(4)]}
    out = np.zeros((n, 10), np.int32)
    for i in range(n):
        cands = []        # (cost, order key, result)
        for r in range(n_rf):
            cands.append((J[i, r, 0], (0, r), [0, -1, -1, -1, -1, r, r, r, r]))
        for r1, r2 in itertools.product(range(n_rf), repeat=2):
            cands.append((J[i, r1, 1] + J[i, r2, 2], (1, r1, r2), [1, -1, -1, -1, -1, r1, r1, r2, r2]))
            cands.append((J[i, r1, 3] + J[i, r2, 4], (2, r1, r2), [2, -1, -1, -1, -1, r1, r2, r1, r2]))
        per_s = []
        for s in range(4):
            opts = [(sum(J[i, r, p] for p in sub_parts[t](s)), (t, r)) for t in range(4) for r in range(n_rf)]
            per_s.append(opts)
        for combo in itertools.product(*per_s):
            cost = sum(c for c, _ in combo)
            key = (3,) + tuple(x for _, tr in combo for x in tr)
            cands.append((cost, key, [3] + [tr[0] for _, tr in combo] + [tr[1] for _, tr in combo]))
        cost, key, res = min(cands, key=lambda c: (c[0], c[1]))
        out[i, :9] = res
        out[i, 9] = cost
    return out


def satd4_blocks(D):
    """SATD of an [h, w] difference array (h, w multiples of 4): sum over 4x4 blocks of
    (sum |Hd D Hd^T| + 1) >> 1 with the Sylvester Hadamard matrix from scipy (rows in
    another order than the oracle's; the abs-sum does not depend on it)"""
    from scipy.linalg import hadamard
    Hd = hadamard(4)
    tot = 0
    for by in range(0, D.shape[0], 4):
        for bx in range(0, D.shape[1], 4):
            T = Hd @ D[by:by + 4, bx:bx + 4] @ Hd.T
            tot += (int(np.abs(T).sum()) + 1) >> 1
    return tot


def sme_satd(cf, rfs, mvs, S, lam=0):
    H, W = cf.shape
    mbc, mbr = -(-W // 16), -(-H // 16)
    Wp, Hp = 16 * mbc, 16 * mbr
    pad = S // 2 + 8
    pitch, rows = Wp + 2 * pad, Hp + 2 * pad
    cfp = _edge(cf, ((0, Hp - H), (0, Wp - W)))
    parts = partitions()
    qmvs = np.zeros_like(mvs)
    out = np.zeros(mvs.shape[:3], np.uint16)
    for r, rf in enumerate(rfs):
        P = planes(rf, pad, pitch, rows).astype(np.int64)
        for o in range(mbr * mbc):
            mby, mbx = divmod(o, mbc)
            for p, (ox, oy, w, h) in enumerate(parts):
                x0, y0 = 16 * mbx + ox, 16 * mby + oy
                blk = cfp[y0:y0 + h, x0:x0 + w]

                def cost(vx, vy):
                    ph = 4 * (vy & 3) + (vx & 3)
                    yy, xx = y0 + (vy >> 2) + pad, x0 + (vx >> 2) + pad
                    d = satd4_blocks(blk - P[ph, yy:yy + h, xx:xx + w])
                    return d + lam * (se_bits(vx) + se_bits(vy)), d

                c = (4 * int(mvs[o, r, p, 0]), 4 * int(mvs[o, r, p, 1]))
                (best, bd), bv = cost(*c), c
                for ring_step in (2, 1):
                    ctr = bv
                    for sx, sy in RING1:
                        v = (ctr[0] + ring_step * sx, ctr[1] + ring_step * sy)
                        j, d = cost(*v)
                        if j < best:
                            best, bd, bv = j, d, v
                qmvs[o, r, p] = bv
                out[o, r, p] = bd
    return qmvs, out


# ---------------------------------------------------- G21 predicted-MV centre --

def me_pmv(cf, rfs, S, lam, pmv, max_pmv):
    """brute force with an integer-pel predictor p per (MB, RF), clamped to +-max_pmv:
    candidates p + (dx, dy), lexicographic (SAD + lam*R(4(mv - p)), rank(dx, dy)) minimum"""
    H, W = cf.shape
    R = S // 2
    mbc, mbr = -(-W // 16), -(-H // 16)
    Wp, Hp = 16 * mbc, 16 * mbr
    cfp = _edge(cf, ((0, Hp - H), (0, Wp - W)))
    m = R + 1 + max_pmv
    d = np.arange(-R, R)
    DX, DY = np.meshgrid(d, d)
    rank = rank_closed_form(DX, DY).ravel()
    rate = np.array([lam * (se_bits(4 * x) + se_bits(4 * y)) for x, y in zip(DX.ravel(), DY.ravel())])
    pmv = np.clip(np.asarray(pmv, np.int64).reshape(mbr * mbc, len(rfs), 2), -max_pmv, max_pmv)
    parts = partitions()
    mvs = np.zeros((mbr * mbc, len(rfs), 41, 2), np.int16)
    sads = np.zeros((mbr * mbc, len(rfs), 41), np.uint16)
    for r, rf in enumerate(rfs):
        rfp = _edge(rf, ((m, m + Hp - H), (m, m + Wp - W)))
        for o in range(mbr * mbc):
            mby, mbx = divmod(o, mbc)
            px, py = int(pmv[o, r, 0]), int(pmv[o, r, 1])
            for p, (ox, oy, w, h) in enumerate(parts):
                x0, y0 = 16 * mbx + ox, 16 * mby + oy
                blk = cfp[y0:y0 + h, x0:x0 + w]
                cand = np.array([np.abs(blk - rfp[y0 + py + dy + m:y0 + py + dy + m + h,
                                                  x0 + px + dx + m:x0 + px + dx + m + w]).sum()
                                 for dy, dx in zip(DY.ravel(), DX.ravel())])
                best = np.lexsort((rank, cand + rate))[0]
                mvs[o, r, p] = (px + DX.ravel()[best], py + DY.ravel()[best])
                sads[o, r, p] = cand[best]
    return mvs, sads
