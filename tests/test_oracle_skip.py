"""Pins for the oracle's reduction approximation of the stencil loops
(NEXT-3; §3.3.3: loop step x N, result x N, temporary
zeroed before the loop) and its extended tuner.

* == scipy.ndimage.correlate(mode="nearest") with the perforated kernel
  (weights N_y*N_x*w on the executed rows/columns, zero elsewhere);
* rate 1 == exact; closed forms (mean filters: a rate equal to K keeps only
  the corner tap, K*K * 1/K^2 = 1 -> a shifted copy of the image; constant
  images scale by N*ceil(K/N)/K per skipped axis); separable == dense outer
  product; brute force on 8x8 images;
* the extended tuner: hand-derived candidate order, a constant-image pin
  (mean 9x9, reduction only -> skip_both 3, the first rate whose
  executed-count x rate equals 9), i.i.d. noise -> exact at TOQ 0.95.
"""
import numpy as np
import pytest
from scipy import ndimage

import workloads as W
from workloads import filters as F
from workloads import images


def corr(x, w):
    return ndimage.correlate(np.asarray(x, np.float64), np.asarray(w, np.float64), mode="nearest")


def perforated(w, ny, nx):
    ky, kx = w.shape
    ny, nx = min(ny, ky), min(nx, kx)
    out = np.zeros((ky, kx), np.float64)
    out[::ny, ::nx] = ny * nx * w.astype(np.float64)[::ny, ::nx]
    return out


DENSE = [F.gaussian(3), F.mean(5), F.conv(7, seed=3), F.conv(9), F.conv_signed(5), F.conv(5, seed=4, ky=3)]


@pytest.mark.parametrize("wi", range(len(DENSE)))
@pytest.mark.parametrize("ny,nx", [(1, 1), (2, 1), (1, 2), (2, 2), (3, 3), (4, 1), (1, 5), (9, 9)])
def test_vs_scipy_perforated(O, wi, ny, nx):
    w = DENSE[wi]
    x = W.frames(2, 29, 41, 3)
    got = O.stencil_skip_xy(x, w, ny, nx)
    pk = perforated(w, ny, nx)
    for f in range(2):
        np.testing.assert_allclose(got[f], corr(x[f], pk), rtol=1e-12, atol=1e-9)


def test_rate1_is_exact(O):
    x = W.frames(2, 30, 30, 1)
    for w in DENSE:
        np.testing.assert_allclose(O.stencil_skip_xy(x, w, 1, 1), O.stencil_exact(x, w), rtol=1e-13, atol=1e-10)


@pytest.mark.parametrize("k", [3, 5, 7])
def test_rate_k_is_a_shift(O, k):
    x = images.random_integers((1, 20, 23), 4).astype(np.float32)
    r = k // 2
    got = O.stencil_skip_xy(x, F.mean(k), k, k)[0]
    yy = np.clip(np.arange(20) - r, 0, 19)
    xx = np.clip(np.arange(23) - r, 0, 22)
    expect = x[0][np.ix_(yy, xx)].astype(np.float64) * (k * k * np.float32(1.0 / (k * k)))
    np.testing.assert_allclose(got, expect, rtol=1e-6)


@pytest.mark.parametrize("k,n", [(5, 2), (9, 3), (9, 4), (7, 2), (3, 2)])
def test_constant_image_scaling(O, k, n):
    x = np.full((1, 16, 16), 50.0, np.float32)
    ex = -(-k // n)  # executed iterations per axis
    scale = (n * ex / k) ** 2
    np.testing.assert_allclose(O.stencil_skip_xy(x, F.mean(k), n, n), 50.0 * scale * (k * k * np.float32(1 / (k * k))),
                               rtol=1e-6)


@pytest.mark.parametrize("ny,nx", [(1, 1), (2, 1), (1, 3), (4, 4), (17, 2)])
def test_separable_equals_dense_outer(O, ny, nx):
    wy, wx = F.separable(17, seed_y=1, seed_x=2)
    x = W.frames(1, 40, 52, 2)
    dense = np.outer(wy.astype(np.float64), wx.astype(np.float64))
    np.testing.assert_allclose(O.stencil_skip_xy(x, (wy, wx), ny, nx)[0], corr(x[0], perforated(dense, ny, nx)),
                               rtol=1e-12, atol=1e-9)


@pytest.mark.parametrize("k", [3, 5, 7])
def test_bruteforce_8x8(O, k):
    rng = np.random.default_rng(k)
    x = rng.integers(0, 256, size=(8, 8)).astype(np.float32)
    w = rng.uniform(-1, 1, size=(k, k)).astype(np.float32)
    r = k // 2
    for ny in range(1, k + 2):
        for nx in range(1, k + 2):
            got = O.stencil_skip_xy(x, w, ny, nx)
            sy, sx = min(ny, k), min(nx, k)
            for y in range(8):
                for xx in range(8):
                    tot = 0.0
                    for i in range(-r, r + 1, sy):
                        inner = 0.0
                        for j in range(-r, r + 1, sx):
                            inner += float(w[i + r, j + r]) * float(x[min(max(y + i, 0), 7), min(max(xx + j, 0), 7)])
                        tot += sx * inner
                    assert abs(got[y, xx] - sy * tot) <= 1e-9 * (1 + abs(sy * tot))


def test_candidate_order_hand_derived(O):
    # 3x3 dense, reduction only: rates 2..2 -> skip_both 2 (2x2 = 4 taps), skip_row 2 (2x3), skip_col 2 (3x2)
    assert O.tune_candidates_ex(3, 3, False, 2) == [("skip_both", 2), ("skip_row", 2), ("skip_col", 2)]
    # 5x5 dense, both families: centre2 (1 tap), skip_both 3 (2x2=4), row2/col2 (5), centre1 (9),
    # skip_both 2 (3x3=9, scheme id 3 after centre 0), skip_row 3 (2x5=10), skip_col 3, row1/col1 (15),
    # skip_row 2 (3x5=15, id 4 after row 1 / col 2), skip_col 2
    assert O.tune_candidates_ex(5, 5, False, 3) == [
        ("center", 2), ("skip_both", 3), ("row", 2), ("col", 2), ("center", 1), ("skip_both", 2),
        ("skip_row", 3), ("skip_col", 3), ("row", 1), ("col", 1), ("skip_row", 2), ("skip_col", 2)]
    # 1x5: only the column loop can be skipped
    assert O.tune_candidates_ex(1, 5, False, 2) == [("skip_col", 3), ("skip_col", 2)]
    assert O.tune_candidates_ex(3, 3, False, 1) == O.tune_candidates(3, 3)


def test_tuner_constant_image_pin(O):
    x = np.full((2, 30, 30), 80.0, np.float32)
    r = O.tune_ex(x, F.mean(9), 1 - 1e-6, "mre", flags=2)
    assert (r["scheme"], r["reach"]) == ("skip_both", 3)


def test_tuner_noise_falls_back(O):
    x = W.uniform_noise(96, 96, 5)[None]
    r = O.tune_ex(x, F.mean(5), 0.95, "mre", flags=2)
    assert r["scheme"] == "exact"


def test_tuner_flags1_equals_tune(O):
    x = W.frames(3, 64, 96, 0)
    for w, m in [(F.gaussian(3), "mre"), (F.conv(9), "l2")]:
        for toq in (0.8, 0.9, 0.95):
            a = O.tune_ex(x, w, toq, m, flags=1)
            b = O.tune(x, w, toq, m)
            assert (a["scheme"], a["reach"], a["quality"]) == (b["scheme"], b["reach"], b["quality"])
