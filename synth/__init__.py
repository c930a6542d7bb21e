"""Seeded synthetic star fields shaped like the paper's workloads.

This module holds none of the method's arithmetic (no brightness, PSF, ROI or binning): it only draws star
catalogues -- sub-pixel positions and magnitudes -- and names the benchmark configurations.  It is the one module both
the fp64 oracle tests and the CUDA path's tests/bench use.

Randomness is a counter-based SplitMix64: value i of stream s under seed k is ``mix64(base(k, s) + (i+1)*GAMMA)``,
so any prefix or sub-range of a field can be regenerated independently.  Doubles are rounded to fp32; a coordinate
that rounds up to W (or H) is clamped to the largest fp32 below it.

Paper shapes: stars have "a magnitude within the range of 0~15 and the coordinate in image plane",
are "generated randomly", images are 1024x1024 with 2^5..2^17 stars or 8192 stars,
and Fig. 2 shows 2252 stars on 1024x1024.  BASELINE.json adds the B200-scale configs C1..C5 and the
north-star frame T; SURVEY.md §8(d) gives the generator recipe used here.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, asdict

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _mix64(z: np.ndarray) -> np.ndarray:
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def _base(seed: int, stream: int) -> np.uint64:
    with np.errstate(over="ignore"):
        s = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) * np.uint64(0x100000001B3) + np.uint64(stream) * GAMMA
    return _mix64(np.array([s], dtype=np.uint64))[0]


def u64(seed: int, stream: int, start: int, count: int) -> np.ndarray:
    """Raw SplitMix64 outputs [start, start+count) of (seed, stream)."""
    i = np.arange(start + 1, start + count + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _mix64(_base(seed, stream) + i * GAMMA)


def uniform01(seed: int, stream: int, start: int, count: int) -> np.ndarray:
    """Doubles in [0, 1) with 53 random bits."""
    return (u64(seed, stream, start, count) >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def _f32_below(v: np.ndarray, hi: float) -> np.ndarray:
    out = v.astype(np.float32)
    top = np.nextafter(np.float32(hi), np.float32(0))
    return np.where(out >= np.float32(hi), top, out).astype(np.float32)


@dataclass(frozen=True)
class Field:
    x: np.ndarray
    y: np.ndarray
    mag: np.ndarray

    @property
    def n(self) -> int:
        return int(self.x.shape[0])

    def aos(self) -> np.ndarray:
        """The paper's star record {mag, posX, posY} as an (n, 3) float32 array."""
        return np.ascontiguousarray(np.stack([self.mag, self.x, self.y], axis=1).astype(np.float32))


def uniform_field(n: int, W: int, H: int, seed: int, mag_lo: float = 0.0, mag_hi: float = 15.0) -> Field:
    """Positions U[0,W) x U[0,H), magnitudes U[mag_lo, mag_hi)."""
    x = _f32_below(uniform01(seed, 0, 0, n) * W, W)
    y = _f32_below(uniform01(seed, 1, 0, n) * H, H)
    m = _f32_below(mag_lo + uniform01(seed, 2, 0, n) * (mag_hi - mag_lo), mag_hi)
    return Field(x, y, m)


def clustered_field(n: int, W: int, H: int, seed: int, n_clusters: int = 64, background: float = 0.10,
                    mag_lo: float = 0.0, mag_hi: float = 15.0) -> Field:
    """C4 recipe: n_clusters centres U[0.1W,0.9W) x U[0.1H,0.9H); each star is uniform background with
    probability ``background``, else centre + N(0, (W/128)^2) per axis; candidates outside the image are rejected."""
    cx = 0.1 * W + uniform01(seed, 10, 0, n_clusters) * 0.8 * W
    cy = 0.1 * H + uniform01(seed, 11, 0, n_clusters) * 0.8 * H
    sd = W / 128.0
    xs, ys = [], []
    have, start = 0, 0
    while have < n:
        k = max(1024, int((n - have) * 1.25))
        u_bg = uniform01(seed, 12, start, k)
        u_cl = uniform01(seed, 13, start, k)
        u1 = uniform01(seed, 14, start, k)
        u2 = uniform01(seed, 15, start, k)
        ub_x = uniform01(seed, 16, start, k)
        ub_y = uniform01(seed, 17, start, k)
        r = np.sqrt(-2.0 * np.log1p(-u1))                      # Box-Muller, 1-u1 in (0, 1]
        gx, gy = r * np.cos(2 * math.pi * u2), r * np.sin(2 * math.pi * u2)
        c = np.minimum((u_cl * n_clusters).astype(np.int64), n_clusters - 1)
        bg = u_bg < background
        px = np.where(bg, ub_x * W, cx[c] + sd * gx)
        py = np.where(bg, ub_y * H, cy[c] + sd * gy)
        ok = (px >= 0) & (px < W) & (py >= 0) & (py < H)
        xs.append(px[ok])
        ys.append(py[ok])
        have += int(ok.sum())
        start += k
    x = _f32_below(np.concatenate(xs)[:n], W)
    y = _f32_below(np.concatenate(ys)[:n], H)
    m = _f32_below(mag_lo + uniform01(seed, 2, 0, n) * (mag_hi - mag_lo), mag_hi)
    return Field(x, y, m)


def adversarial_field(n: int, W: int, H: int, R: int, seed: int, with_nonfinite: bool = True) -> Field:
    """Edge cases for the ROI origin, clipping and culling: integer and half-integer coordinates and their fp32
    neighbours, stars just off every border, far-off stars, and (optionally) NaN / +-inf entries.  Bright (m in
    [0, 2)) so every star matters at the parity tolerance."""
    u = [uniform01(seed, 20 + j, 0, n) for j in range(6)]
    kind = np.minimum((u[0] * 8).astype(np.int64), 7)
    base_x = np.floor(u[1] * (W + 2 * R)) - R
    base_y = np.floor(u[2] * (H + 2 * R)) - R
    frac_choices = np.array([0.0, 0.5, 0.25, 0.75], dtype=np.float64)
    fx = frac_choices[np.minimum((u[3] * 4).astype(np.int64), 3)]
    fy = frac_choices[np.minimum((u[4] * 4).astype(np.int64), 3)]
    x = (base_x + fx).astype(np.float32)
    y = (base_y + fy).astype(np.float32)
    # nudge some to the fp32 neighbours of the grid points
    up = kind == 1
    dn = kind == 2
    x = np.where(up, np.nextafter(x, np.float32(np.inf)), x)
    x = np.where(dn, np.nextafter(x, np.float32(-np.inf)), x)
    y = np.where(kind == 3, np.nextafter(y, np.float32(np.inf)), y)
    y = np.where(kind == 4, np.nextafter(y, np.float32(-np.inf)), y)
    # plain random sub-pixel positions over the extended area
    rnd = kind == 5
    x = np.where(rnd, ((u[5] * (W + 2 * R)) - R).astype(np.float32), x)
    y = np.where(rnd, ((u[3] * (H + 2 * R)) - R).astype(np.float32), y)
    # far-off stars
    far = kind == 6
    x = np.where(far & (u[5] < 0.5), np.float32(-1e6), x)
    y = np.where(far & (u[5] >= 0.5), np.float32(3e7), y)
    m = (u[5] * 2.0).astype(np.float32)
    if with_nonfinite and n >= 8:
        x = x.copy(); y = y.copy(); m = m.copy()
        x[3] = np.float32(np.nan)
        y[5] = np.float32(np.inf)
        m[7] = np.float32(-np.inf)
    return Field(x.astype(np.float32), y.astype(np.float32), m.astype(np.float32))


@dataclass(frozen=True)
class Config:
    """One benchmark / parity configuration (BASELINE.json configs)."""
    name: str
    W: int
    H: int
    n: int
    R: int
    sigma: float
    kind: str            # "uniform" | "clustered"
    seed: int

    def field(self, n: int | None = None, mag_lo: float = 0.0, mag_hi: float = 15.0) -> Field:
        n = self.n if n is None else n
        if self.kind == "clustered":
            return clustered_field(n, self.W, self.H, self.seed, mag_lo=mag_lo, mag_hi=mag_hi)
        return uniform_field(n, self.W, self.H, self.seed, mag_lo=mag_lo, mag_hi=mag_hi)

    def as_dict(self) -> dict:
        return asdict(self)


def sigma_for(R: int) -> float:
    """Where a config gives no sigma: sigma = R/6, so the ROI spans +-3 sigma (reading R4)."""
    return R / 6.0


CONFIGS = {
    # BASELINE.json configs[0]: 1024x1024, 1,000 uniform stars, R=5, sigma=1.0
    "C1": Config("C1", 1024, 1024, 1000, 5, 1.0, "uniform", 1),
    # configs[1]: 2048x2048, 20,000 stars, R=9, sigma=1.5
    "C2": Config("C2", 2048, 2048, 20000, 9, 1.5, "uniform", 2),
    # configs[2]: 4096x4096 star-count sweep at R=11 (the point at 2^20 stars; others via field(n=...))
    "C3": Config("C3", 4096, 4096, 1 << 20, 11, sigma_for(11), "uniform", 3),
    # configs[3]: 4096x4096, 100K clustered stars, R sweep 3..63 (R=15 point; others via with_R)
    "C4": Config("C4", 4096, 4096, 100000, 15, sigma_for(15), "clustered", 4),
    # configs[4]: 16384x16384, 10M stars, R=15, banded over GPUs
    "C5": Config("C5", 16384, 16384, 10_000_000, 15, sigma_for(15), "uniform", 5),
    # north-star frame: 4096x4096, 1M stars, R=15, 1 GPU
    "T": Config("T", 4096, 4096, 1_000_000, 15, sigma_for(15), "uniform", 6),
    # Fig. 2: 1024x1024 with 2252 stars
    "fig2": Config("fig2", 1024, 1024, 2252, 11, 1.0, "uniform", 7),
}

C3_COUNTS = [1 << k for k in range(10, 21)] + [1_000_000]
C4_RADII = [3, 5, 7, 9, 11, 15, 21, 31, 47, 63]


def with_R(cfg: Config, R: int) -> Config:
    return Config(f"{cfg.name}_R{R}", cfg.W, cfg.H, cfg.n, R, sigma_for(R), cfg.kind, cfg.seed)


def bench_gain(sigma: float, bits: int = 8) -> float:
    """Benchmark A (reading R1): an m=0 star centred on a pixel peaks at full scale 2^bits - 1."""
    return 2.0 * math.pi * sigma * sigma * (2 ** bits - 1)
