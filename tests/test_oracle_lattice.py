"""Pins for the oracle's global-lattice stencil (NEXT-1, reading G;
PAPER.md L350-356 "accesses a subset of values in the input array and
replicates that subset to construct an approximate version of the array").

* the per-axis map g equals the hand table tests/golden/lattice_map.txt;
* the stencil equals scipy.ndimage.correlate(mode="nearest") applied to the
  array rebuilt from the accessed rows/columns (library routine);
* invariants: reach 0 == exact; an image already constant over each lattice
  group is reproduced exactly; no output depends on a non-accessed pixel;
  constant images are fixed points; separable == dense outer product.
"""
import os

import numpy as np
import pytest
from scipy import ndimage

import workloads as W
from workloads import images
from workloads import filters as F

GOLD = os.path.join(os.path.dirname(__file__), "golden", "lattice_map.txt")


def _rows():
    out = []
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        v = [int(t) for t in line.split()]
        out.append((v[0], v[1], v[2:]))
    return out


@pytest.mark.parametrize("length,d,expect", _rows())
def test_hand_table(O, length, d, expect):
    assert list(O.lattice_map(length, d)) == expect


@pytest.mark.parametrize("length", [1, 2, 5, 9, 16, 31])
@pytest.mark.parametrize("d", [0, 1, 2, 3, 4, 8])
def test_map_properties(O, length, d):
    g = O.lattice_map(length, d)
    s = 2 * d + 1
    assert g[0] == 0
    assert np.all(np.diff(g) >= 0)                       # monotone
    assert np.all(g % s == 0) and np.all(g < length)     # accessed coords are in range
    assert np.all(g[g] == g)                             # idempotent
    last = s * ((length - 1) // s)
    inner = np.arange(length) <= last + d
    assert np.all(np.abs(g - np.arange(length))[inner] <= d)  # within the reach, up to the tail


def corr(x, w):
    return ndimage.correlate(np.asarray(x, np.float64), np.asarray(w, np.float64), mode="nearest")


DENSE = [F.gaussian(3), F.mean(5), F.conv(7, seed=3), F.conv(9), F.conv_signed(5), F.conv(5, seed=4, ky=3)]


@pytest.mark.parametrize("wi", range(len(DENSE)))
@pytest.mark.parametrize("dy,dx", [(0, 0), (1, 0), (0, 1), (1, 1), (2, 0), (3, 3), (4, 0)])
def test_vs_scipy_on_rebuilt_array(O, wi, dy, dx):
    w = DENSE[wi]
    x = W.frames(2, 37, 50, 7)
    gy, gx = O.lattice_map(37, dy), O.lattice_map(50, dx)
    got = O.stencil_lattice_xy(x, w, dy, dx)
    for f in range(2):
        xt = x[f][np.ix_(gy, gx)]
        np.testing.assert_allclose(got[f], corr(xt, w), rtol=1e-12, atol=1e-9)


def test_reach0_is_exact(O):
    x = W.frames(2, 40, 33, 3)
    for w in DENSE:
        np.testing.assert_array_equal(O.stencil_lattice_xy(x, w, 0, 0), O.stencil_exact(x, w))


def test_group_constant_image_is_reproduced(O):
    """Rows replicated over every lattice group: X~ == X, so the row scheme is exact."""
    rng = np.random.default_rng(5)
    h, w_, d = 41, 30, 2
    s = 2 * d + 1
    base = rng.integers(16, 236, size=(h, w_)).astype(np.float32)
    x = np.empty_like(base)
    for y in range(h):  # every row takes its nearest multiple of s, the tail the last
        a = s * int(np.floor(y / s + 0.5))
        x[y] = base[min(a, s * ((h - 1) // s))]
    for w in DENSE:
        np.testing.assert_allclose(O.stencil_lattice(x, w, "row", d), O.stencil_exact(x, w), rtol=0, atol=1e-9)


def test_non_accessed_pixels_do_not_matter(O):
    x = images.random_integers((19, 23), 9).astype(np.float32)
    w = F.conv(5, seed=8)
    for dy, dx in [(1, 0), (0, 2), (1, 1)]:
        gy, gx = O.lattice_map(19, dy), O.lattice_map(23, dx)
        base = O.stencil_lattice_xy(x, w, dy, dx)
        acc_y, acc_x = set(gy.tolist()), set(gx.tolist())
        for y in range(19):
            for xx in range(23):
                z = x.copy()
                z[y, xx] += 50.0
                out = O.stencil_lattice_xy(z, w, dy, dx)
                if y in acc_y and xx in acc_x:
                    continue
                np.testing.assert_array_equal(out, base)


def test_accessed_pixel_matters(O):
    x = images.random_integers((19, 23), 10).astype(np.float32)
    w = F.mean(3)
    base = O.stencil_lattice_xy(x, w, 1, 0)
    z = x.copy()
    z[3, 4] += 9.0  # row 3 is accessed (multiple of 3)
    assert not np.array_equal(O.stencil_lattice_xy(z, w, 1, 0), base)


def test_constant_fixed_point(O):
    x = np.full((2, 25, 31), 77.0, dtype=np.float32)
    for w in (F.gaussian(3), F.mean(5), F.conv(9)):
        np.testing.assert_allclose(O.stencil_lattice_xy(x, w, 2, 1), 77.0, rtol=1e-6)


@pytest.mark.parametrize("dy,dx", [(0, 0), (1, 0), (0, 3), (2, 2)])
def test_separable_equals_dense_outer(O, dy, dx):
    wy, wx = F.separable(7)
    x = W.frames(1, 33, 45, 2)
    dense = np.outer(wy.astype(np.float64), wx.astype(np.float64))
    np.testing.assert_allclose(O.stencil_lattice_xy(x, (wy, wx), dy, dx),
                               corr(x[0][np.ix_(O.lattice_map(33, dy), O.lattice_map(45, dx))], dense)[None],
                               rtol=1e-12, atol=1e-9)


# ---- lattice tuner pins ---------------------------------------------------

def test_tuner_constant_image_takes_sparsest(O):
    x = np.full((2, 40, 40), 99.0, dtype=np.float32)
    r = O.tune_lattice(x, F.mean(5), 1 - 1e-6, "mre")
    assert (r["scheme"], r["reach"]) == ("row", 4)


def test_tuner_y_constant_image_takes_sparsest(O):
    row = images.random_integers((1, 64), 3).astype(np.float32)
    x = np.repeat(row, 50, axis=0)[None]
    r = O.tune_lattice(x, F.conv(5, seed=2), 1 - 1e-9, "l2")
    assert (r["scheme"], r["reach"]) == ("row", 4)
    assert all(abs(q - 1.0) < 1e-6 for q in r["qualities"])


def test_tuner_noise_falls_back_to_exact(O):
    x = W.uniform_noise(96, 96, 5)[None]
    r = O.tune_lattice(x, F.mean(5), 0.95, "mre")
    assert (r["scheme"], r["reach"], r["quality"]) == ("exact", 0, 1.0)


def test_tuner_first_passing_and_monotone(O):
    x = W.frames(2, 96, 128, 0)
    w = F.gaussian(3)
    qs = O.tune_lattice(x, w, 2.0, "mre")["qualities"]  # nothing passes: all four qualities
    assert qs[0] <= qs[1] <= qs[2] <= qs[3] < 1.0  # sparser rows, lower quality (on these images)
    for toq in (0.8, 0.9, 0.95, 0.99):
        r = O.tune_lattice(x, w, toq, "mre")
        passing = [k for k, q in enumerate(qs) if q >= toq]
        if passing:
            assert (r["scheme"], r["reach"]) == ("row", 4 - passing[0])
            assert r["quality"] == qs[passing[0]]
        else:
            assert r["scheme"] == "exact"
