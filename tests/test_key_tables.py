"""The ME key tables libfeves_me.so builds on the host (me_key_tables, no GPU needed) against the
oracle's spiral enumeration (G4, pin P10) -- DESIGN.md §6 "key-sum aggregation".

What must hold for the GPU argmin to equal the oracle's strict-< spiral-order search:
- the dense rank orders candidates exactly as the oracle's spiral rank does;
- inv maps the dense rank back to (dx, dy), covering the SA once;
- key-sum: a partition of n 4x4 blocks carries n * r in the low 16 bits, so n * r < 2^16 for
  every rank the kernel sums (S <= 64: the dense rank; S = 128: the rank inside a quadrant);
- S = 128 quadrant mode: local ranks follow the spiral order inside each quadrant and glob maps
  them back to the dense rank;
- with a rate term (G18) the addend is lambda * R(4dx, 4dy) * 2^15 + dense rank.
"""
import ctypes

import numpy as np
import pytest

import oracle as orc


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    L = pkg.lib()
    p = ctypes.POINTER(ctypes.c_uint32)
    L.me_key_tables.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, p, p, p]
    L.me_key_tables.restype = ctypes.c_int
    return L


def tables(lib, S, inclusive=0, lam=0):
    Sc = S + inclusive
    Sp = (Sc + 3) & ~3
    e = np.zeros(Sc * Sp, np.uint32)
    inv = np.zeros((S + 1) * (S + 1), np.uint32)
    glob = np.zeros(4 * 4096, np.uint32)
    p = ctypes.POINTER(ctypes.c_uint32)
    rc = lib.me_key_tables(S, inclusive, lam, e.ctypes.data_as(p), inv.ctypes.data_as(p), glob.ctypes.data_as(p))
    assert rc == 0
    return e.reshape(Sc, Sp), inv, glob


def unpack(v):
    def s16(x):
        return x - 0x10000 if x & 0x8000 else x
    return s16(v & 0xFFFF), s16(v >> 16)


def se_bits(v):   # Exp-Golomb se(v) length, written out (G18)
    k = 2 * v - 1 if v > 0 else -2 * v
    n = 0
    while (k + 1) >> (n + 1):
        n += 1
    return 2 * n + 1


@pytest.mark.parametrize("S,inclusive", [(4, 0), (16, 0), (18, 0), (32, 0), (64, 0), (64, 1), (128, 0)])
def test_dense_rank_is_spiral_order(lib, S, inclusive):
    R = S // 2
    Sc = S + inclusive
    e, inv, glob = tables(lib, S, inclusive)
    cands = [unpack(int(v)) for v in inv[: Sc * Sc]]
    assert len(set(cands)) == Sc * Sc                                   # the SA, once
    assert all(-R <= dx <= Sc - 1 - R and -R <= dy <= Sc - 1 - R for dx, dy in cands)
    assert cands == orc.spiral_candidates(S, bool(inclusive))           # dense rank == O1's visiting order
    if S == 128 and not inclusive:
        return                                                          # quadrant mode: next test
    for r, (dx, dy) in enumerate(cands):
        assert e[dx + R, dy + R] == r
    if S <= 64 and not inclusive:
        assert 16 * (Sc * Sc - 1) < 1 << 16                             # key-sum: no carry into SAD


def test_quadrant_tables_s128(lib):
    S, R = 128, 64
    e, inv, glob = tables(lib, S)
    seen = [[] for _ in range(4)]
    for r in range(S * S):
        dx, dy = unpack(int(inv[r]))
        q = 2 * (dy >= 0) + (dx >= 0)
        loc = int(e[dx + R, dy + R])
        assert loc < 4096 and 16 * loc < 1 << 16                        # per-quadrant key-sum bound
        assert glob[q * 4096 + loc] == r                                # local -> dense rank
        seen[q].append(loc)
    for q in range(4):                                                  # each quadrant: 0..4095 in spiral order
        assert seen[q] == list(range(4096))


@pytest.mark.parametrize("S,lam", [(16, 4), (32, 25), (128, 9)])
def test_rate_term_addend(lib, S, lam):
    R = S // 2
    e, inv, _ = tables(lib, S, 0, lam)
    for r in range(0, S * S, 7):
        dx, dy = unpack(int(inv[r]))
        assert e[dx + R, dy + R] == lam * (se_bits(4 * dx) + se_bits(4 * dy)) * (1 << 15) + r


def test_bad_arguments(lib):
    p = ctypes.POINTER(ctypes.c_uint32)
    buf = np.zeros(1 << 16, np.uint32)
    q = buf.ctypes.data_as(p)
    for args in [(2, 0, 0), (130, 0, 0), (15, 0, 0), (16, 2, 0), (16, 0, -1), (16, 0, 2001)]:
        assert lib.me_key_tables(*args, q, q, q) == -1
    assert lib.me_key_tables(16, 0, 0, None, q, q) == -1
