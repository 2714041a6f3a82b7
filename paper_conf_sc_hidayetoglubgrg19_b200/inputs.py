"""Seeded synthetic inputs shared by the tests, the bench and the oracle legs.

This module holds NONE of the method's arithmetic (no tracing, ordering, SpMV or CG).  It only
makes inputs with the structure of the paper's workloads (DESIGN.md section 4 "input recipe"):

* ``shepp_logan(n)`` -- the modified Shepp-Logan phantom sampled at pixel centres (reading R17),
  the standard noiseless test object; the paper's datasets (ADS1-4 are synthetic) are
  reconstructions of phantom-like objects on full-field-of-view parallel-beam scans.
* ``uniform(n, seed)`` / ``normal(n, seed)`` -- seeded random vectors for SpMV throughput and the
  adjoint identity (values do not change the access pattern).
* ``CONFIGS`` -- BASELINE.json's five configurations (N, projections, channels).

Pixel (row i, col j) of an N x N tomogram covers [j - N/2, j + 1 - N/2) x [i - N/2, i + 1 - N/2)
(reading R3); the natural index is i*N + j.
"""
from __future__ import annotations

import numpy as np

#: BASELINE.json "configs" (N, projections M, channels C), in order.
CONFIGS = {
    1: (64, 90, 64),
    2: (256, 360, 256),
    3: (1024, 1500, 1024),
    4: (2048, 2400, 2048),
    5: (11293, 360, 11293),
}

#: seed rule of SURVEY 8(d): seed = 0x5EED00 + cfg
def seed_for(cfg: int) -> int:
    return 0x5EED00 + int(cfg)


# Modified Shepp-Logan ellipses (A, a, b, x0, y0, phi_degrees), Toft's modification.
_SHEPP_LOGAN = (
    (1.0, 0.69, 0.92, 0.0, 0.0, 0.0),
    (-0.8, 0.6624, 0.874, 0.0, -0.0184, 0.0),
    (-0.2, 0.11, 0.31, 0.22, 0.0, -18.0),
    (-0.2, 0.16, 0.41, -0.22, 0.0, 18.0),
    (0.1, 0.21, 0.25, 0.0, 0.35, 0.0),
    (0.1, 0.046, 0.046, 0.0, 0.1, 0.0),
    (0.1, 0.046, 0.046, 0.0, -0.1, 0.0),
    (0.1, 0.046, 0.023, -0.08, -0.605, 0.0),
    (0.1, 0.023, 0.023, 0.0, -0.606, 0.0),
    (0.1, 0.023, 0.046, 0.06, -0.605, 0.0),
)


def shepp_logan(n: int, dtype=np.float64) -> np.ndarray:
    """N x N modified Shepp-Logan phantom, row-major (row i increases with y)."""
    c = (np.arange(n) + 0.5 - n / 2.0) / (n / 2.0)
    u = c[None, :]  # x from column j
    v = c[:, None]  # y from row i
    img = np.zeros((n, n), np.float64)
    for A, a, b, x0, y0, phi in _SHEPP_LOGAN:
        ph = np.deg2rad(phi)
        cp, sp = np.cos(ph), np.sin(ph)
        xr = (u - x0) * cp + (v - y0) * sp
        yr = -(u - x0) * sp + (v - y0) * cp
        img += A * ((xr * xr) / (a * a) + (yr * yr) / (b * b) <= 1.0)
    return img.astype(dtype).reshape(-1)


def uniform(n: int, seed: int, dtype=np.float32) -> np.ndarray:
    """U[0, 1) vector (seeded)."""
    return np.random.default_rng(seed).random(n).astype(dtype)


def normal(n: int, seed: int, dtype=np.float64) -> np.ndarray:
    """N(0, 1) vector (seeded)."""
    return np.random.default_rng(seed).standard_normal(n).astype(dtype)
