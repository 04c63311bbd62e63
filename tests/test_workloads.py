"""The seeded input generators: determinism, value range and the Fig. 5
calibration (>75% of pixels within 10% of their 8
neighbours)."""
import numpy as np
import pytest

import workloads as W
from workloads import filters as F


@pytest.mark.parametrize("h,w", [(64, 64), (512, 512), (240, 384)])
def test_fig5_calibrated(h, w):
    for seed in (0, 1):
        x = W.image(h, w, seed)
        s = W.fig5_statistic(x)
        assert 0.75 <= s <= 0.80, s
        assert x.dtype == np.float32
        assert x.min() >= 16 and x.max() <= 235
        assert np.all(x == np.rint(x))


def test_deterministic():
    a = W.image(100, 120, 7)
    b = W.image(100, 120, 7)
    assert np.array_equal(a, b)
    assert not np.array_equal(a, W.image(100, 120, 8))
    f = W.frames(3, 50, 60, 4)
    assert np.array_equal(f[1], W.image(50, 60, 5))


def test_periodic_tile_seamless():
    t = W.image(64, 64, 2)
    p = W.periodic(150, 200, tile=64, seed=2)
    assert np.array_equal(p[:64, :64], t)
    assert np.array_equal(p[64:128, 128:192], t)


def test_filters():
    assert np.array_equal(F.gaussian(3) * 16, np.array([[1, 2, 1], [2, 4, 2], [1, 2, 1]], np.float32))
    assert abs(float(F.conv(9).astype(np.float64).sum()) - 1.0) < 1e-6
    wy, wx = F.separable(7)
    assert wy.shape == (7,) and wx.shape == (7,) and not np.array_equal(wy, wx)
    assert F.named("mean5")[1].shape == (5, 5)
