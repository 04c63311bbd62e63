"""Pins for the oracle's HotSpot steps (NEXT-4; Table 1, 3x3 tiles
L1916-1920; update of reading S25):

* one exact step == T + c (P + correlate(T, 5-point Laplacian with gx, gy,
  mode="nearest") + gz (Tamb - T)) (scipy library routine);
* T = Tamb, P = 0 is a fixed point of every scheme;
* uniform T and P: the closed-form geometric approach to Tamb + P/gz;
* centre scheme (full collapse): the per-pixel closed form without neighbours;
* row scheme: only the horizontal Laplacian remains (scipy correlate1d), the
  column scheme the vertical one;
* k iterations == k single steps.
"""
import numpy as np
import pytest
from scipy import ndimage

from workloads import hotspot as H

PRM = dict(c=1.0, gx=0.1, gy=0.07, gz=0.002, tamb=320.0)


def step_ref(t, p, prm, vert=True, horiz=True):
    t = t.astype(np.float64)
    k = np.zeros((3, 3))
    if vert:
        k[0, 1] = k[2, 1] = prm["gy"]
        k[1, 1] -= 2 * prm["gy"]
    if horiz:
        k[1, 0] = k[1, 2] = prm["gx"]
        k[1, 1] -= 2 * prm["gx"]
    lap = ndimage.correlate(t, k, mode="nearest")
    return t + prm["c"] * (p.astype(np.float64) + lap + prm["gz"] * (prm["tamb"] - t))


def test_one_step_vs_scipy(O):
    t, p = H.frames(1, 37, 52, 3)
    np.testing.assert_allclose(O.hotspot(t[0], p[0], PRM), step_ref(t[0], p[0], PRM), rtol=1e-13, atol=1e-10)


@pytest.mark.parametrize("dy,dx", [(0, 0), (1, 0), (0, 1), (1, 1), (2, 5)])
def test_ambient_fixed_point(O, dy, dx):
    t = np.full((2, 20, 30), PRM["tamb"], np.float32)
    p = np.zeros_like(t)
    np.testing.assert_allclose(O.hotspot(t, p, PRM, dy, dx, 7), PRM["tamb"], rtol=0, atol=1e-9)


@pytest.mark.parametrize("dy,dx", [(0, 0), (1, 0), (1, 1)])
def test_uniform_closed_form(O, dy, dx):
    t0, p0, k = 330.0, 0.5, 9
    t = np.full((16, 16), t0, np.float32)
    p = np.full((16, 16), p0, np.float32)
    tinf = PRM["tamb"] + p0 / PRM["gz"]
    expect = tinf + (t0 - tinf) * (1 - PRM["c"] * PRM["gz"]) ** k
    np.testing.assert_allclose(O.hotspot(t, p, PRM, dy, dx, k), expect, rtol=1e-12)


def test_centre_is_pointwise(O):
    t, p = H.frames(1, 24, 31, 5)
    got = O.hotspot(t[0], p[0], PRM, 1, 1, 4)
    ref = t[0].astype(np.float64)
    for _ in range(4):
        ref = ref + PRM["c"] * (p[0] + PRM["gz"] * (PRM["tamb"] - ref))
    np.testing.assert_allclose(got, ref, rtol=1e-13)


def test_row_and_col_schemes_drop_one_laplacian(O):
    t, p = H.frames(1, 29, 33, 8)
    np.testing.assert_allclose(O.hotspot(t[0], p[0], PRM, 1, 0), step_ref(t[0], p[0], PRM, vert=False),
                               rtol=1e-13, atol=1e-10)
    np.testing.assert_allclose(O.hotspot(t[0], p[0], PRM, 0, 1), step_ref(t[0], p[0], PRM, horiz=False),
                               rtol=1e-13, atol=1e-10)


def test_iterations_compose(O):
    t, p = H.frames(1, 21, 26, 2)
    a = O.hotspot(t[0], p[0], PRM, 0, 0, 5)
    ref = t[0].astype(np.float64)
    for _ in range(5):
        ref = step_ref(ref, p[0], PRM)
    np.testing.assert_allclose(a, ref, rtol=1e-12)
