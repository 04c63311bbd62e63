"""Pins for the oracle's exact and approximate stencils.

* exact == scipy.ndimage.correlate(mode="nearest") (library routine; clamp-to-
  edge borders, reading S7; correlation, reading S8);
* literal per-window substitution == correlate with the folded kernel (an
  identity: the substituted tile dotted with w equals the representatives
  dotted with the summed weights);
* closed forms (3x3 Gaussian and 5x5 mean collapses, quadratic probe),
  invariants (reach 0, constant images, tile-local substitution), impulse
  response, and brute force on 8x8 images.
"""
import numpy as np
import pytest
from scipy import ndimage

import workloads as W
from workloads import filters as F


def fold(O, w, dy, dx):
    """Folded kernel on the full K_y x K_x grid (test-side, from the oracle's
    pinned index maps)."""
    ky, kx = w.shape
    my = O.index_map(ky // 2, dy) + ky // 2
    mx = O.index_map(kx // 2, dx) + kx // 2
    wf = np.zeros((ky, kx), dtype=np.float64)
    for i in range(ky):
        for j in range(kx):
            wf[my[i], mx[j]] += float(w[i, j])
    return wf


def corr(x, w):
    return ndimage.correlate(np.asarray(x, np.float64), np.asarray(w, np.float64), mode="nearest")


FILTERS = [
    ("gauss3", F.gaussian(3)),
    ("mean5", F.mean(5)),
    ("conv7", F.conv(7, seed=3)),
    ("conv9", F.conv(9)),
    ("signed5", F.conv_signed(5)),
    ("rect3x7", F.conv(7, seed=11, ky=3)),
    ("rect9x1", F.conv(1, seed=12, ky=9)),
]


@pytest.mark.parametrize("name,w", FILTERS)
def test_exact_vs_scipy(O, name, w):
    x = W.image(37, 53, 1)
    e = O.stencil_exact(x, w)
    np.testing.assert_allclose(e, corr(x, w), rtol=1e-12, atol=1e-9)


def test_exact_batch_frames_independent(O):
    x = W.frames(3, 20, 17, 5)
    w = F.conv(5, seed=9)
    e = O.stencil_exact(x, w)
    for k in range(3):
        np.testing.assert_allclose(e[k], corr(x[k], w), rtol=1e-12, atol=1e-9)


@pytest.mark.parametrize("name,w", FILTERS)
def test_approx_vs_folded_scipy(O, name, w):
    x = W.image(33, 41, 2)
    ky, kx = w.shape
    for dy in range(0, ky // 2 + 2):
        for dx in range(0, kx // 2 + 2):
            a = O.stencil_approx_xy(x, w, dy, dx)
            np.testing.assert_allclose(a, corr(x, fold(O, w, dy, dx)), rtol=1e-12, atol=1e-9,
                                       err_msg=f"{name} dy={dy} dx={dx}")


@pytest.mark.parametrize("name,w", FILTERS)
def test_reach0_is_exact(O, name, w):
    x = W.image(29, 31, 3)
    np.testing.assert_array_equal(O.stencil_approx_xy(x, w, 0, 0), O.stencil_exact(x, w))


def test_gaussian3_full_collapse_closed_forms(O):
    """3x3 binomial Gaussian at reach 1: row -> horizontal [1/4 1/2 1/4],
    column -> vertical [1/4 1/2 1/4], centre -> identity (sum w = 1)."""
    x = W.image(40, 40, 4)
    w = F.gaussian(3)
    k = np.array([0.25, 0.5, 0.25])
    row = O.stencil_approx(x, w, "row", 1)
    col = O.stencil_approx(x, w, "col", 1)
    cen = O.stencil_approx(x, w, "center", 1)
    np.testing.assert_allclose(row, ndimage.correlate1d(x.astype(np.float64), k, axis=1, mode="nearest"),
                               rtol=1e-15)
    np.testing.assert_allclose(col, ndimage.correlate1d(x.astype(np.float64), k, axis=0, mode="nearest"),
                               rtol=1e-15)
    np.testing.assert_allclose(cen, x.astype(np.float64), rtol=1e-15)
    # reach 2 saturates to reach 1 on a 3x3 tile
    np.testing.assert_array_equal(O.stencil_approx(x, w, "center", 2), cen)


def test_mean5_closed_forms(O):
    """5x5 mean, reach 1: per-axis groups (1,3,1) -> centre weights 1/25
    (corners), 3/25 (edges), 9/25 (centre) at offsets {-2,0,2}^2; reach 2 ->
    row = 1-D horizontal box 1/5, centre = identity."""
    x = W.image(30, 30, 6)
    w = F.mean(5)
    wc = np.zeros((5, 5))
    g = {0: 1.0, 2: 3.0, 4: 1.0}
    for a, ga in g.items():
        for b, gb in g.items():
            wc[a, b] = ga * gb * float(np.float32(1 / 25))
    np.testing.assert_allclose(O.stencil_approx(x, w, "center", 1), corr(x, wc), rtol=1e-14)
    box = np.full(5, 5 * float(np.float32(1 / 25)))
    np.testing.assert_allclose(O.stencil_approx(x, w, "row", 2),
                               ndimage.correlate1d(x.astype(np.float64), box, axis=1, mode="nearest"),
                               rtol=1e-14)
    np.testing.assert_allclose(O.stencil_approx(x, w, "center", 2),
                               25 * float(np.float32(1 / 25)) * x.astype(np.float64), rtol=1e-14)


@pytest.mark.parametrize("name,w", FILTERS[:5])
def test_constant_image_fixed_point(O, name, w):
    x = np.full((2, 16, 19), 97.0, dtype=np.float32)
    s = float(np.sum(w.astype(np.float64)))
    ky, kx = w.shape
    for dy in range(ky // 2 + 1):
        for dx in range(kx // 2 + 1):
            np.testing.assert_allclose(O.stencil_approx_xy(x, w, dy, dx), 97.0 * s, rtol=1e-14)


@pytest.mark.parametrize("name,w", FILTERS)
def test_row_scheme_exact_on_y_constant(O, name, w):
    """Rows that are all alike: replacing a row by another changes nothing."""
    xr = W.image(1, 45, 7)
    x = np.repeat(xr, 23, axis=0)
    e = O.stencil_exact(x, w)
    for d in range(1, w.shape[0] // 2 + 2):
        np.testing.assert_allclose(O.stencil_approx(x, w, "row", d), e, rtol=1e-13)
    xc = np.repeat(W.image(45, 1, 8), 23, axis=1)
    ec = O.stencil_exact(xc, w)
    for d in range(1, w.shape[1] // 2 + 2):
        np.testing.assert_allclose(O.stencil_approx(xc, w, "col", d), ec, rtol=1e-13)


@pytest.mark.parametrize("name,w", FILTERS)
def test_impulse_response_is_flipped_folded_kernel(O, name, w):
    ky, kx = w.shape
    for dy, dx in [(0, 0), (1, 0), (0, 1), (1, 1), (2, 3)]:
        x = np.zeros((ky + 6, kx + 6), dtype=np.float32)
        cy, cx = ky // 2 + 3, kx // 2 + 3
        x[cy, cx] = 1.0
        a = O.stencil_approx_xy(x, w, dy, dx)
        wf = fold(O, w, dy, dx)
        # out(q - (a, b)) = w'[a][b]  => window around the impulse = flipped w'
        win = a[cy - ky // 2:cy + ky // 2 + 1, cx - kx // 2:cx + kx // 2 + 1]
        np.testing.assert_allclose(win, wf[::-1, ::-1], rtol=1e-15, atol=0)


def test_non_accessed_element_does_not_matter(O):
    """Changing X at an offset of p that is not accessed leaves A(p) unchanged;
    changing an accessed one does change it (tile-local substitution)."""
    w = F.conv(7, seed=21)
    x = W.image(25, 25, 9)
    p = (12, 12)
    for dy, dx in [(1, 1), (2, 0), (0, 3), (1, 2)]:
        my = O.index_map(3, dy)
        mx = O.index_map(3, dx)
        base = O.stencil_approx_xy(x, w, dy, dx)[p]
        for i in range(-3, 4):
            for j in range(-3, 4):
                x2 = x.copy()
                x2[p[0] + i, p[1] + j] += 50.0
                changed = O.stencil_approx_xy(x2, w, dy, dx)[p] != base
                accessed = (i in set(my.tolist())) and (j in set(mx.tolist()))
                assert changed == accessed, (dy, dx, i, j)


@pytest.mark.parametrize("k", [3, 5, 7, 9])
def test_quadratic_probe(O, k):
    """X = (y - y0)^2 in the interior: E - A = sum_i u_i (i^2 - m(i)^2) with
    u_i = sum_j w_ij (row / centre schemes); 0 for the column scheme."""
    w = F.mean(k) if k != 9 else F.gaussian(9)
    h, wd = 40, 30
    yy = np.arange(h, dtype=np.float64)[:, None] - 20
    x = np.repeat(yy ** 2, wd, axis=1).astype(np.float32)
    r = k // 2
    u = w.astype(np.float64).sum(axis=1)
    i = np.arange(-r, r + 1)
    inner = (slice(r, h - r), slice(r, wd - r))
    e = O.stencil_exact(x, w)
    for d in range(1, r + 1):
        m = O.index_map(r, d)
        expect = float(np.sum(u * (i ** 2 - m ** 2)))
        for scheme in ("row", "center"):
            a = O.stencil_approx(x, w, scheme, d)
            np.testing.assert_allclose((e - a)[inner], expect, rtol=1e-12, atol=1e-9)
        a = O.stencil_approx(x, w, "col", d)
        np.testing.assert_allclose((e - a)[inner], 0.0, atol=1e-9)
    # the worked number: mean 5x5, row scheme, reach 1 -> E - A = 0.4
    if k == 5:
        a = O.stencil_approx(x, w, "row", 1)
        np.testing.assert_allclose((e - a)[inner], 0.4, rtol=1e-6)


def _brute(x, w, my, mx):
    """Materialise every substituted window with fancy indexing and dot it."""
    h, wd = x.shape
    ky, kx = w.shape
    ys = np.clip(np.arange(h)[:, None, None, None] + my[None, None, :, None], 0, h - 1)
    xs = np.clip(np.arange(wd)[None, :, None, None] + mx[None, None, None, :], 0, wd - 1)
    win = x.astype(np.float64)[ys, xs]          # [h, w, ky, kx]
    return np.einsum("hwij,ij->hw", win, w.astype(np.float64))


@pytest.mark.parametrize("k", [1, 3, 5, 7])
def test_bruteforce_8x8(O, k):
    """All schemes and reaches 0..r+1 on 8x8 random integer images, where the
    borders dominate (clamp semantics)."""
    w = F.conv(k, seed=100 + k) if k > 1 else np.ones((1, 1), np.float32)
    r = k // 2
    for seed in range(3):
        x = W.images.random_integers((8, 8), seed)
        for scheme in ("exact", "row", "col", "center"):
            for d in range(0, r + 2):
                dy, dx = O.scheme_reaches(scheme, d)
                my = O.index_map(r, dy)
                mx = O.index_map(r, dx)
                np.testing.assert_allclose(O.stencil_approx(x, w, scheme, d), _brute(x, w, my, mx),
                                           rtol=1e-13, atol=1e-10)


@pytest.mark.parametrize("ky,kx", [(7, 7), (3, 5), (9, 1), (1, 9)])
def test_separable_equals_dense_outer(O, ky, kx):
    """Two-pass separable approx with (dy, dx) == dense approx with wy (x) wx."""
    wy = F.conv(1, seed=31, ky=ky).ravel() if ky > 1 else np.ones(1, np.float32)
    wx = F.conv(kx, seed=32, ky=1).ravel()
    dense = np.outer(wy.astype(np.float64), wx.astype(np.float64))
    x = W.image(26, 34, 10)
    for dy in range(ky // 2 + 1):
        for dx in range(kx // 2 + 1):
            s = O.stencil_sep(x, wy, wx, dy, dx)
            # dense oracle on the fp64 outer product: compare with scipy fold
            np.testing.assert_allclose(s, corr(x, fold(O, dense, dy, dx)), rtol=1e-12)


def test_rejects_even_and_empty(O):
    x = W.image(8, 8, 0)
    with pytest.raises(ValueError):
        O.stencil_exact(x, np.ones((2, 3), np.float32))
    with pytest.raises(ValueError):
        O.stencil_approx_xy(x, F.gaussian(3), -1, 0)
