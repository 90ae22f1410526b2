"""CPU oracle for the FEVES ME -> INT -> SME hot path.  TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  The product package
``paper_conf_icpp_ilicmrs14_b200`` never imports it, and the two share no code.

This module is argument marshalling (ctypes) over ``feves_oracle.c``; every
arithmetic step of the method lives in that C file, which cites the passage of
/root/reference/PAPER.md it follows.  Oracle functions and their pins
(tests/test_oracle_*.py):

  spiral_rank        G4                P1, P10 (closed form vs enumeration)
  me                 O1  (P:6)         P1 hand-computed, P2, P3, P4, P9 NumPy brute force
  me(lam>0), sme(lam>0)  G18 (f4)      P12 hand-computed rate pins, P13 NumPy brute force
  mode_decision      O4  (f2)    P14 closed forms, P13 NumPy enumeration
  sme(satd=True)     G20 (f4)          P15 Hadamard closed forms, P13 NumPy (scipy Hadamard) SME
  sample/int_planes  O2  (P:6)  P5 closed forms + golden, P6, P7, P9
  sme                O3  (P:6)   P2, P8 (incl. half-pel synthetic), P9
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "feves_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

N_PART = 41


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc -O2, OpenMP over MBs only)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-Wall",
                               "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i = ctypes.c_int
        L.oracle_me.argtypes = [P, P, i, i, i, i, i, P, i, P, P, i]
        L.oracle_me_rd.argtypes = [P, P, i, i, i, i, i, i, P, i, P, P, i]
        L.oracle_sme.argtypes = [P, P, i, i, i, P, i, P, P, P, i]
        L.oracle_sme_rd.argtypes = [P, P, i, i, i, i, P, i, P, P, P, i]
        L.oracle_sme_ex.argtypes = [P, P, i, i, i, i, i, P, i, P, P, P, i]
        L.oracle_satd_q.argtypes = [P, P, i, i, i, i, i, i, i, i]
        L.oracle_satd_q.restype = ctypes.c_long
        L.oracle_mode_decision.argtypes = [P, P, i, i, i, P]
        L.oracle_me_pmv.argtypes = [P, P, i, i, i, i, i, i, P, i, P, i, P, P, i]
        L.oracle_sme_pmv.argtypes = [P, P, i, i, i, i, i, P, i, P, i, P, P, P, i]
        L.oracle_mode_decision_pmv.argtypes = [P, P, i, i, i, P, i, P]
        L.oracle_mv_bits.argtypes = [i, i]
        L.oracle_mv_bits.restype = i
        L.oracle_int_planes.argtypes = [P, i, i, i, i, i, i, i, P, i]
        for fn in ("oracle_sample", "oracle_b1", "oracle_h1", "oracle_j1",
                   "oracle_j_horizontal_first", "oracle_ref_px"):
            getattr(L, fn).argtypes = [P, i, i, i, i]
            getattr(L, fn).restype = i
        L.oracle_spiral_rank.argtypes = [i, i]
        L.oracle_spiral_candidates.argtypes = [i, i, P, P]
        L.oracle_spiral_candidates.restype = i
        L.oracle_partition_geom.argtypes = [i, P]
        L.oracle_num_threads.restype = i
        _lib = L
    return _lib


def _u8(a):
    a = np.ascontiguousarray(a, dtype=np.uint8)
    assert a.ndim == 2
    return a


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def _ptr_array(frames):
    arr = (ctypes.c_void_p * len(frames))(*[f.ctypes.data for f in frames])
    return arr


def num_threads() -> int:
    return lib().oracle_num_threads()


def partition_geom(p: int):
    out = np.zeros(4, np.int32)
    lib().oracle_partition_geom(p, _ptr(out))
    return tuple(int(v) for v in out)


def spiral_rank(dx: int, dy: int) -> int:
    return lib().oracle_spiral_rank(dx, dy)


def spiral_candidates(S: int, sa_inclusive: bool = False):
    """The SA's candidates (dx, dy) in the order O1 visits them (G1, G4)."""
    n = (S + int(sa_inclusive)) ** 2
    dx, dy = np.zeros(n, np.int32), np.zeros(n, np.int32)
    assert lib().oracle_spiral_candidates(S, int(sa_inclusive), _ptr(dx), _ptr(dy)) == n
    return list(zip(dx.tolist(), dy.tolist()))


def all_mbs(W: int, H: int, row_begin: int = 0, row_end: int | None = None):
    mb_cols, mb_rows = (W + 15) // 16, (H + 15) // 16
    row_end = mb_rows if row_end is None else row_end
    return np.arange(row_begin * mb_cols, row_end * mb_cols, dtype=np.int32)


def _pmv(pmv, n, n_rf):
    """G21 predictor array int16 [n, n_rf, 2] (or None = the zero predictor)."""
    if pmv is None:
        return None
    return np.ascontiguousarray(pmv, np.int16).reshape(n, n_rf, 2)


def me(cf, rfs, sa_range: int, mb_list=None, sa_inclusive: bool = False, threads: int = 0, lam: int = 0,
       pmv=None, max_pmv: int = 0):
    """O1 (lam > 0: cost J = SAD + lam * R(mv - p), G18; pmv: integer-pel predictor p per
    (frame MB, RF) [mb_rows * mb_cols, n_rf, 2], each component clamped to +-max_pmv, the SA
    centred on p, G21). Returns (mvs int16 [n_mb, n_rf, 41, 2], sads uint16 [n_mb, n_rf, 41])
    -- the SAD of the chosen MV."""
    cf = _u8(cf)
    rfs = [_u8(r) for r in rfs]
    H, W = cf.shape
    mb_list = all_mbs(W, H) if mb_list is None else np.ascontiguousarray(mb_list, np.int32)
    n = len(mb_list)
    mvs = np.zeros((n, len(rfs), N_PART, 2), np.int16)
    sads = np.zeros((n, len(rfs), N_PART), np.uint16)
    pm = _pmv(pmv, ((W + 15) // 16) * ((H + 15) // 16), len(rfs))
    rc = lib().oracle_me_pmv(_ptr(cf), _ptr_array(rfs), W, H, sa_range, len(rfs), int(sa_inclusive), int(lam),
                             None if pm is None else _ptr(pm), int(max_pmv),
                             _ptr(mb_list), n, _ptr(mvs), _ptr(sads), threads)
    if rc != 0:
        raise ValueError("oracle_me: bad arguments")
    return mvs, sads


def sme(cf, rfs, in_mvs, mb_list=None, threads: int = 0, lam: int = 0, satd: bool = False,
        pmv=None, max_pmv: int = 0):
    """O3 (lam > 0: cost J = D + lam * R(qmv - 4p), G18, G21 (pmv as for me); satd: D = Hadamard SATD, G20).
    in_mvs int16 [n_mb, n_rf, 41, 2] full-pel. Returns (qmvs, distortions)."""
    cf = _u8(cf)
    rfs = [_u8(r) for r in rfs]
    H, W = cf.shape
    mb_list = all_mbs(W, H) if mb_list is None else np.ascontiguousarray(mb_list, np.int32)
    n = len(mb_list)
    in_mvs = np.ascontiguousarray(in_mvs, np.int16).reshape(n, len(rfs), N_PART, 2)
    qmvs = np.zeros((n, len(rfs), N_PART, 2), np.int16)
    sads = np.zeros((n, len(rfs), N_PART), np.uint16)
    pm = _pmv(pmv, ((W + 15) // 16) * ((H + 15) // 16), len(rfs))
    rc = lib().oracle_sme_pmv(_ptr(cf), _ptr_array(rfs), W, H, len(rfs), int(lam), int(satd),
                              None if pm is None else _ptr(pm), int(max_pmv), _ptr(mb_list), n,
                              _ptr(in_mvs), _ptr(qmvs), _ptr(sads), threads)
    if rc != 0:
        raise ValueError("oracle_sme: bad arguments")
    return qmvs, sads


def satd_q(cf, rf, x0, y0, w, h, vx, vy) -> int:
    """G20 SATD of the w x h block at (x0, y0) against rf at quarter-pel offset (vx, vy)."""
    cf, rf = _u8(cf), _u8(rf)
    return int(lib().oracle_satd_q(_ptr(cf), _ptr(rf), cf.shape[1], cf.shape[0], x0, y0, w, h, vx, vy))


def mv_bits(qx: int, qy: int) -> int:
    """G18 R(mv): se(v) Exp-Golomb bits of the quarter-pel MV components."""
    return lib().oracle_mv_bits(qx, qy)


def mode_decision(qmvs, sads, lam: int, pmv=None, max_pmv: int = 0):
    """O4: per MB [mb_type, sub_type x4, ref per 8x8 x4, cost] int32 [n_mb, 10].
    pmv (G21): [n_mb, n_rf, 2] predictor of each listed MB; J uses R(qmv - 4p)."""
    qmvs = np.ascontiguousarray(qmvs, np.int16)
    sads = np.ascontiguousarray(sads, np.uint16)
    n, n_rf = sads.shape[0], sads.shape[1]
    out = np.zeros((n, 10), np.int32)
    pm = _pmv(pmv, n, n_rf)
    if lib().oracle_mode_decision_pmv(_ptr(qmvs), _ptr(sads), n, n_rf, int(lam), None if pm is None else _ptr(pm),
                                      int(max_pmv), _ptr(out)) != 0:
        raise ValueError("oracle_mode_decision: bad arguments")
    return out


def sample(rf, X: int, Y: int) -> int:
    rf = _u8(rf)
    return lib().oracle_sample(_ptr(rf), rf.shape[1], rf.shape[0], X, Y)


def raw(name: str, rf, x: int, y: int) -> int:
    """Pre-clip intermediates b1/h1/j1, 'j_hfirst', or 'ref' (clamped integer sample)."""
    rf = _u8(rf)
    fn = {"b1": "oracle_b1", "h1": "oracle_h1", "j1": "oracle_j1",
          "j_hfirst": "oracle_j_horizontal_first", "ref": "oracle_ref_px"}[name]
    return getattr(lib(), fn)(_ptr(rf), rf.shape[1], rf.shape[0], x, y)


def sf_layout(W: int, H: int, sa_range: int):
    """G11 SF geometry: (pad, pitch, rows) with pad = ceil((R+4)/16)*16."""
    R = sa_range // 2
    pad = -(-(R + 4) // 16) * 16
    Wp, Hp = -(-W // 16) * 16, -(-H // 16) * 16
    return pad, Wp + 2 * pad, Hp + 2 * pad


def int_planes(rf, pad: int, pitch: int, rows: int, row_begin: int = 0, row_end: int | None = None,
               threads: int = 0):
    """O2 planes [16, rows, pitch] u8, plane origin at integer position (-pad, -pad)."""
    rf = _u8(rf)
    out = np.zeros((16, rows, pitch), np.uint8)
    row_end = rows if row_end is None else row_end
    rc = lib().oracle_int_planes(_ptr(rf), rf.shape[1], rf.shape[0], pad, pitch, rows,
                                 row_begin, row_end, _ptr(out), threads)
    if rc != 0:
        raise ValueError("oracle_int_planes: bad arguments")
    return out
