"""Seeded filter weights for the paper's stencil workloads (inputs, not method).

* Gaussian: binomial [1 2 1]^T [1 2 1] / 16 generalised to K taps (reading S15
  in DESIGN.md; the paper gives no sigma, Table 1).
* Mean: 1/K^2 everywhere (Table 1 "Mean Filter").
* Convolution: seeded U(0, 1) weights normalised to sum 1 in fp64, then cast to
  fp32 (reading S16; the paper's ConvSep weights are not given, L1650).

All weights are returned as fp32 numpy arrays, row-major [ky, kx] (dense) or
two 1-D arrays (separable).
"""
from __future__ import annotations

from math import comb

import numpy as np


def binomial_1d(k: int) -> np.ndarray:
    c = np.array([comb(k - 1, i) for i in range(k)], dtype=np.float64)
    return (c / c.sum()).astype(np.float32)


def gaussian(k: int = 3) -> np.ndarray:
    b = binomial_1d(k).astype(np.float64)
    return np.outer(b, b).astype(np.float32)


def mean(k: int = 5) -> np.ndarray:
    return np.full((k, k), 1.0 / (k * k), dtype=np.float32)


def conv(k: int = 9, seed: int = 1234, ky: int | None = None) -> np.ndarray:
    ky = k if ky is None else ky
    rng = np.random.default_rng(seed)
    w = rng.uniform(0.0, 1.0, size=(ky, k))
    return (w / w.sum()).astype(np.float32)


def conv_signed(k: int = 5, seed: int = 77) -> np.ndarray:
    """Signed weights (sum 1): exercises cancellation in parity tolerances."""
    rng = np.random.default_rng(seed)
    w = rng.uniform(-1.0, 1.0, size=(k, k))
    w[k // 2, k // 2] += 1.0 - w.sum()
    return w.astype(np.float32)


def separable(k: int = 7, seed_y: int = 4321, seed_x: int = 8765):
    """Two independent seeded normalised 1-D filters (w_y, w_x)."""
    out = []
    for s in (seed_y, seed_x):
        rng = np.random.default_rng(s)
        v = rng.uniform(0.0, 1.0, size=k)
        out.append((v / v.sum()).astype(np.float32))
    return out[0], out[1]


def named(name: str):
    """Filters of the BASELINE.json configs: returns ("dense", w) or ("sep", (wy, wx))."""
    if name == "gauss3":
        return "dense", gaussian(3)
    if name == "mean5":
        return "dense", mean(5)
    if name == "sep7":
        return "sep", separable(7)
    if name == "conv9":
        return "dense", conv(9)
    raise KeyError(name)
