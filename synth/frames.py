"""Seeded synthetic 8-bit luma frames.

gen_tex   textured content in global sub-pixel motion: a continuous sum of 8
          random 2-D sinusoids (periods 8..128 px) scaled to [16, 235],
          evaluated at (x - t*vx, y - t*vy) so the motion is exact without any
          interpolation filter, plus N(0, 2^2) per-frame noise.
gen_noise i.i.d. uniform u8 (worst case for SAD magnitudes; timing is
          content-independent under FSBM).
gen_flat  gen_tex with 25% of the MBs replaced by one constant per MB (the
          same in every frame): many exactly tied candidates (G4 tie-break).
gen_shifted  CF(x,y) = RF(clamp(x+u), clamp(y+v)): a known global integer shift.

IPPP (G15): frame t is the CF; RF k (ref_idx k) is frame t-1-k.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass(frozen=True)
class Config:
    name: str
    width: int
    height: int
    n_rf: int
    sa_range: int
    path: str          # "me" or "me+int+sme"
    gpus: tuple        # GPU counts the config is quoted at
    baseline_index: int


# BASELINE.json `configs`, in order.
CONFIGS = {
    "cif": Config("cif", 352, 288, 1, 16, "me", (1,), 0),
    "1080p_sa32": Config("1080p_sa32", 1920, 1080, 1, 32, "me", (1,), 1),
    "1080p_sa64_4rf": Config("1080p_sa64_4rf", 1920, 1080, 4, 64, "me+int+sme", (1,), 2),
    "1080p_shard": Config("1080p_shard", 1920, 1080, 4, 64, "me+int+sme", (2, 4, 8), 3),
    "2160p_sa128": Config("2160p_sa128", 3840, 2160, 4, 128, "me+int+sme", (8,), 4),
}


def _tex_field(W, H, t, seed, velocity=(1.25, -0.75)):
    rng = np.random.default_rng(seed)
    y, x = np.mgrid[0:H, 0:W].astype(np.float64)
    xs = x - t * velocity[0]
    ys = y - t * velocity[1]
    acc = np.zeros((H, W))
    amps = rng.uniform(0.3, 1.0, 8)
    for k in range(8):
        period = rng.uniform(8.0, 128.0)
        theta = rng.uniform(0, np.pi)
        phase = rng.uniform(0, 2 * np.pi)
        acc += amps[k] * np.sin(2 * np.pi / period * (np.cos(theta) * xs + np.sin(theta) * ys) + phase)
    acc /= amps.sum()                      # in [-1, 1]
    return 125.5 + 109.5 * acc             # in [16, 235]


def gen_tex(W, H, t, seed, noise_sigma=2.0):
    f = _tex_field(W, H, t, seed)
    rng = np.random.default_rng((seed, t, 7))
    f = f + rng.normal(0.0, noise_sigma, f.shape)
    return np.clip(np.rint(f), 0, 255).astype(np.uint8)


def gen_noise(W, H, t, seed):
    rng = np.random.default_rng((seed, t, 11))
    return rng.integers(0, 256, (H, W), dtype=np.uint8)


def gen_flat(W, H, t, seed, frac=0.25):
    f = gen_tex(W, H, t, seed)
    rng = np.random.default_rng((seed, 13))          # same MBs + values in every frame
    mbc, mbr = -(-W // 16), -(-H // 16)
    mask = rng.random((mbr, mbc)) < frac
    vals = rng.integers(16, 236, (mbr, mbc))
    for r, c in zip(*np.nonzero(mask)):
        f[16 * r:16 * r + 16, 16 * c:16 * c + 16] = vals[r, c]
    return f


def gen_shifted(rf, u, v):
    """CF(x, y) = RF(clamp(x+u), clamp(y+v)) -- plain clamped indexing."""
    H, W = rf.shape
    ys = np.clip(np.arange(H) + v, 0, H - 1)
    xs = np.clip(np.arange(W) + u, 0, W - 1)
    return np.ascontiguousarray(rf[ys][:, xs])


_GEN = {"tex": gen_tex, "noise": gen_noise, "flat": gen_flat}


def ippp_sequence(W, H, n_frames, seed, kind="tex"):
    g = _GEN[kind]
    return [g(W, H, t, seed) for t in range(n_frames)]


def make_workload(cfg: Config | str, kind="tex", seed=None, t_cf=None):
    """Returns (cf, [rf_0 .. rf_{n_rf-1}]) with rf_k = frame t_cf-1-k (G15).

    Seeds default to 1000 + the BASELINE.json config index.
    """
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    seed = 1000 + cfg.baseline_index if seed is None else seed
    t_cf = cfg.n_rf if t_cf is None else t_cf
    g = _GEN[kind]
    cf = g(cfg.width, cfg.height, t_cf, seed)
    rfs = [g(cfg.width, cfg.height, t_cf - 1 - k, seed) for k in range(cfg.n_rf)]
    return cf, rfs
