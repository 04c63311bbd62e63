"""Seeded synthetic HotSpot inputs (NEXT-4; Table 1: HotSpot,
1024x1024).  Input generators only -- none of the method's arithmetic.

The paper's Rodinia inputs (temperature and power traces of a floorplan) are
not available.  Recipe (reading S25):
* temperature: a calibrated 1/f field (images.image) scaled to [323, 343] K;
* power: a floorplan of seeded rectangular blocks with power densities in
  [0, 1] (per-step heating c * P up to 1 K), plus the 1/f field at 10 %;
* coefficients (dimensionless per step): c = 1, gx = gy = 0.1 (an explicit step
  needs c (2 gx + 2 gy) < 1), gz = 0.001, Tamb = 323.
"""
from __future__ import annotations

import numpy as np

from . import images

PARAMS = dict(c=1.0, gx=0.1, gy=0.1, gz=0.001, tamb=323.0)


def temperature(h: int, w: int, seed: int) -> np.ndarray:
    x = images.image(h, w, seed).astype(np.float64)
    return (323.0 + (x - 16.0) / 219.0 * 20.0).astype(np.float32)


def power(h: int, w: int, seed: int, blocks: int = 24) -> np.ndarray:
    rng = np.random.default_rng(seed + 7919)
    p = np.zeros((h, w), np.float64)
    for _ in range(blocks):
        bh, bw = max(1, int(rng.integers(h // 16 + 1, h // 4 + 2))), max(1, int(rng.integers(w // 16 + 1, w // 4 + 2)))
        y0, x0 = int(rng.integers(0, max(1, h - bh))), int(rng.integers(0, max(1, w - bw)))
        p[y0:y0 + bh, x0:x0 + bw] = rng.uniform(0.0, 1.0)
    p += 0.1 * (images.image(h, w, seed + 104729).astype(np.float64) - 16.0) / 219.0
    return p.astype(np.float32)


def frames(n: int, h: int, w: int, seed0: int = 0):
    t = np.stack([temperature(h, w, seed0 + k) for k in range(n)])
    p = np.stack([power(h, w, seed0 + k) for k in range(n)])
    return t, p
