"""Seeded synthetic images shaped like the paper's stencil workloads.

Input generators only: this module holds none of the method's arithmetic (no
stencil, no index map, no quality metric).  It is the one module both the
oracle side (``oracle/``) and the CUDA side (tests, ``bench.py``) consume, so
that both see bit-identical inputs.

Recipe:

* A 2-D Gaussian random field with power spectrum ``|F(f)|^2 ~ f^-beta``,
  ``beta = 2`` (the 1/f amplitude spectrum of natural images), made by shaping
  seeded white noise (numpy ``default_rng(seed)``, PCG64) in the Fourier
  domain, normalised to unit standard deviation.
* ``X = clip(rint(125.5 + a * field + sigma * z), 16, 235)`` with ``z`` seeded
  N(0, 1) sensor noise, ``sigma = 3``; values are integers in [16, 235] stored
  as fp32 (exactly representable, so every consumer sees identical inputs).
* The contrast ``a`` is calibrated per image by bisection so that the paper's
  Fig. 5 adjacency statistic lands at 77.5 % (inside the 75-80 % band): the
  share of pixels whose mean |difference| to their 8 neighbours is below 10 %
  of the pixel ("more than 75% of pixels are less than 10% different",
  PAPER.md L1078-1082 Fig. 5 caption; "more than 70%", L1136-1142 §3.2.1).
  The statistic is evaluated on a seeded sample of <= 262144 interior pixels.

Every frame is a pure function of (h, w, seed).
"""
from __future__ import annotations

import functools

import numpy as np

try:  # scipy's pocketfft takes float32 and threads; numpy's is the fallback
    import scipy.fft as _fft

    def _rfft2(a):
        return _fft.rfft2(a, workers=-1)

    def _irfft2(a, s):
        return _fft.irfft2(a, s=s, workers=-1)
except Exception:  # pragma: no cover
    def _rfft2(a):
        return np.fft.rfft2(a)

    def _irfft2(a, s):
        return np.fft.irfft2(a, s=s)

BETA = 2.0
SIGMA = 3.0
TARGET_FIG5 = 0.775
LO, HI = 16.0, 235.0
_NSAMPLE = 262144
_OFFS8 = [(dy, dx) for dy in (-1, 0, 1) for dx in (-1, 0, 1) if (dy, dx) != (0, 0)]


def fig5_statistic(x: np.ndarray, threshold: float = 0.10) -> float:
    """Share of interior pixels whose mean |X(q) - X(p)| over the 8 neighbours q
    is below ``threshold`` * X(p) (Fig. 5; L1132-1142)."""
    x = np.asarray(x, dtype=np.float64)
    h, w = x.shape
    if h < 3 or w < 3:
        return float("nan")
    c = x[1:-1, 1:-1]
    acc = np.zeros_like(c)
    for dy, dx in _OFFS8:
        acc += np.abs(x[1 + dy:h - 1 + dy, 1 + dx:w - 1 + dx] - c)
    return float(np.mean(acc / 8.0 < threshold * c))


def _field(h: int, w: int, rng: np.random.Generator) -> np.ndarray:
    white = rng.standard_normal((h, w))
    spec = _rfft2(white)
    fy = np.fft.fftfreq(h)[:, None]
    fx = np.fft.rfftfreq(w)[None, :]
    f = np.sqrt(fy * fy + fx * fx)
    f[0, 0] = 1.0
    spec *= f ** (-BETA / 2.0)
    spec[0, 0] = 0.0
    g = _irfft2(spec, (h, w))
    sd = g.std()
    return g / sd if sd > 0 else g


def _compose(a: float, g: np.ndarray, z: np.ndarray) -> np.ndarray:
    return np.clip(np.rint(125.5 + a * g + z), LO, HI)


@functools.lru_cache(maxsize=64)
def _image_cached(h: int, w: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    g = _field(h, w, rng)
    z = rng.standard_normal((h, w)) * SIGMA
    if h >= 3 and w >= 3:
        n = min(_NSAMPLE, (h - 2) * (w - 2))
        ys = rng.integers(1, h - 1, n)
        xs = rng.integers(1, w - 1, n)
        # 3x3 neighbourhoods of the sample, gathered once
        gs = np.stack([g[ys + dy, xs + dx] for dy, dx in [(0, 0)] + _OFFS8])
        zs = np.stack([z[ys + dy, xs + dx] for dy, dx in [(0, 0)] + _OFFS8])
        lo, hi = 0.0, 80.0
        for _ in range(20):
            a = 0.5 * (lo + hi)
            v = _compose(a, gs, zs)
            stat = np.mean(np.abs(v[1:] - v[0]).sum(0) / 8.0 < 0.10 * v[0])
            if stat > TARGET_FIG5:
                lo = a
            else:
                hi = a
        a = 0.5 * (lo + hi)
    else:
        a = 20.0
    img = _compose(a, g, z).astype(np.float32)
    img.setflags(write=False)
    return img


def image(h: int, w: int, seed: int) -> np.ndarray:
    """One calibrated [h, w] fp32 frame (integers in [16, 235])."""
    return _image_cached(int(h), int(w), int(seed)).copy()


def frames(n: int, h: int, w: int, seed0: int = 0) -> np.ndarray:
    """[n, h, w] fp32 batch of frames with seeds seed0 .. seed0+n-1."""
    out = np.empty((n, h, w), dtype=np.float32)
    for k in range(n):
        out[k] = _image_cached(int(h), int(w), int(seed0 + k))
    return out


def periodic(h: int, w: int, tile: int = 4096, seed: int = 0) -> np.ndarray:
    """[h, w] image made by repeating one tile x tile frame.  The FFT field is
    periodic, so the repeat is seamless (config c4's 32768^2 image)."""
    t = _image_cached(tile, tile, int(seed))
    reps = (-(-h // tile), -(-w // tile))
    return np.ascontiguousarray(np.tile(t, reps)[:h, :w])


def uniform_noise(h: int, w: int, seed: int, lo: int = 16, hi: int = 235) -> np.ndarray:
    """i.i.d. uniform integers in [lo, hi] (no spatial correlation), fp32."""
    rng = np.random.default_rng(seed)
    return rng.integers(lo, hi + 1, size=(h, w)).astype(np.float32)


def random_integers(shape, seed: int, lo: int = 0, hi: int = 255) -> np.ndarray:
    """Small-range integer test images (brute-force cases), fp32."""
    rng = np.random.default_rng(seed)
    return rng.integers(lo, hi + 1, size=shape).astype(np.float32)
