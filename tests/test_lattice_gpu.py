"""GPU parity of the global-lattice reading (NEXT-1, reading G;
PAPER.md L350-356) against the oracle's exact stencil on the rebuilt array.

Tolerance as in test_parity_gpu (reading S18): per output
|gpu - oracle| <= 1e-5 * (oracle lattice stencil of |w| on |X|).  The
lattice tuner's decisions must equal the oracle lattice tuner's."""
import numpy as np
import pytest
import torch

import workloads as W
from workloads import filters as F

pytestmark = pytest.mark.gpu

RTOL = 1e-5


@pytest.fixture(scope="module")
def P():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def absw(w):
    return (np.abs(w[0]), np.abs(w[1])) if isinstance(w, tuple) else np.abs(w)


def mkf(P, w):
    return P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)


def check(P, O, x, w, dy, dx, out=None, xd=None):
    f = mkf(P, w)
    g = P.stencil_lattice_xy(dev(x) if xd is None else xd, f, dy, dx, out=out).cpu().numpy()
    o = O.stencil_lattice_xy(x, w, dy, dx)
    bound = RTOL * O.stencil_lattice_xy(np.abs(x), absw(w), dy, dx) + 1e-30
    err = np.abs(g - o)
    assert np.all(err <= bound), (dy, dx, float((err / bound).max()), P.last_kernel())
    return P.last_kernel()


FILTERS = [
    ("gauss3", F.gaussian(3)),
    ("mean5", F.mean(5)),
    ("conv7", F.conv(7, seed=3)),
    ("conv9", F.conv(9)),
    ("signed5", F.conv_signed(5)),
    ("sep7", F.separable(7)),
    ("sep3", F.separable(3, seed_y=5, seed_x=6)),
    ("sep9", F.separable(9, seed_y=7, seed_x=8)),
]


@pytest.mark.parametrize("name,w", FILTERS, ids=[f[0] for f in FILTERS])
@pytest.mark.parametrize("shape", [(2, 77, 300), (1, 257, 516), (3, 40, 128)], ids=["2x77x300", "1x257x516", "3x40x128"])
def test_row_lattice_fast_path(P, O, name, w, shape):
    x = W.frames(*shape, seed0=4)
    for d in (1, 2, 3, 4):
        k = check(P, O, x, w, d, 0)
        assert k.startswith("lattice_dense" if not isinstance(w, tuple) else "lattice_sep"), (d, k)


@pytest.mark.parametrize("name,w", [FILTERS[1], FILTERS[3], FILTERS[5], ("rect3x5", F.conv(5, seed=4, ky=3))],
                         ids=["mean5", "conv9", "sep7", "rect3x5"])
def test_col_and_centre_lattice(P, O, name, w):
    x = W.frames(2, 61, 203, 8)
    for dy, dx in [(0, 1), (0, 3), (1, 1), (2, 2), (4, 1), (6, 0), (0, 7)]:
        check(P, O, x, w, dy, dx)


def test_reach_beyond_fast_path_and_tiny_images(P, O):
    w = F.mean(5)
    for shape in [(1, 1, 1), (1, 2, 3), (2, 5, 5), (1, 9, 700), (1, 700, 9)]:
        x = W.frames(*shape, seed0=2) if min(shape[1:]) >= 3 else np.random.default_rng(0).integers(
            16, 236, size=shape).astype(np.float32)
        for dy, dx in [(1, 0), (5, 0), (0, 2), (3, 3), (20, 20)]:
            check(P, O, x, w, dy, dx)


def test_reach0_is_exact_bitwise(P):
    x = dev(W.frames(2, 100, 160, 1))
    f = P.Filter(F.conv(7, seed=3))
    assert torch.equal(P.stencil_lattice_xy(x, f, 0, 0), P.stencil_exact(x, f))
    assert torch.equal(P.stencil_lattice(x, f, "exact", 3), P.stencil_exact(x, f))


def test_scheme_entry_points(P):
    x = dev(W.frames(1, 90, 128, 6))
    f = P.Filter(F.mean(5))
    assert torch.equal(P.stencil_lattice(x, f, "row", 2), P.stencil_lattice_xy(x, f, 2, 0))
    assert torch.equal(P.stencil_lattice(x, f, "col", 2), P.stencil_lattice_xy(x, f, 0, 2))
    assert torch.equal(P.stencil_lattice(x, f, "center", 2), P.stencil_lattice_xy(x, f, 2, 2))


def test_fast_and_generic_agree(P, O, monkeypatch):
    """The misaligned copy takes the generic lattice kernel; both meet the oracle."""
    w = F.conv(9)
    x = W.frames(2, 150, 336, 30)
    buf = torch.zeros(2 * 150 * 336 + 1, device="cuda")
    mis = buf[1:].view(2, 150, 336)
    mis.copy_(dev(x))
    ob = torch.zeros(2 * 150 * 336 + 1, device="cuda")[1:].view(2, 150, 336)
    for d in (1, 2, 4):
        assert check(P, O, x, w, d, 0).startswith("lattice_dense")
        assert check(P, O, x, w, d, 0, out=ob, xd=mis) == "lattice_generic"


def test_pitched_layout(P, O):
    w = F.mean(5)
    x = W.frames(2, 64, 200, 3)
    big = torch.zeros(2, 70, 256, device="cuda")
    big[:, :64, :200] = dev(x)
    view = big[:, :64, :200]
    out = torch.zeros(2, 70, 256, device="cuda")[:, :64, :200]  # same pitch and frame stride
    g = P.stencil_lattice_xy(view, P.Filter(w), 1, 0, out=out).cpu().numpy()
    o = O.stencil_lattice_xy(x, w, 1, 0)
    assert np.all(np.abs(g - o) <= RTOL * O.stencil_lattice_xy(x, np.abs(w), 1, 0))


def test_halos_rejected(P):
    f = P.Filter(F.mean(5))
    x = torch.rand(1, 70, 64, device="cuda")
    img = P.image_of(x, 3, 3)
    import ctypes as C
    out = torch.empty(1, 64, 64, device="cuda")
    rc = P._lib.paraprox_stencil_lattice_xy(f.handle, 1, 0, P._dp(x, 3), P._dp(out), C.byref(img),
                                            P._stream(None))
    assert rc == P.ERR_INVALID_ARG


TUNE = [("gauss3", F.gaussian(3), "mre", (10, 256, 256)), ("mean5", F.mean(5), "mre", (10, 256, 256)),
        ("conv9", F.conv(9), "l2", (6, 256, 256)), ("sep7", F.separable(7), "l2", (6, 216, 384))]


@pytest.mark.parametrize("name,w,metric,shape", TUNE, ids=[t[0] for t in TUNE])
def test_lattice_tuner_bit_identical(P, O, name, w, metric, shape):
    x = W.frames(*shape, seed0=0)
    f = mkf(P, w)
    xd = dev(x)
    parts = P.tune_lattice_partials(xd, f, metric)
    ref = O.tune_lattice(x, w, 2.0, metric)["qualities"]
    qs = [P.quality_from_partials(parts[3 * k:3 * k + 3], metric) for k in range(4)]
    np.testing.assert_allclose(qs, ref, rtol=0, atol=1e-7)
    for toq in (0.80, 0.90, 0.95, 0.99):
        got = P.tune_lattice(xd, f, toq, metric)
        o = O.tune_lattice(x, w, toq, metric)
        assert got[:2] == (o["scheme"], o["reach"]), (toq, got, o, min(abs(q - toq) for q in ref))
        assert P.tune_lattice_decide(parts, toq, metric) == got


def test_c2_full_frame(P, O):
    """BASELINE configs[1] size, row lattice reach 1 and 2, every output."""
    x = W.image(4096, 4096, 11)[None]
    w = F.mean(5)
    for d in (1, 2):
        assert check(P, O, x, w, d, 0).startswith("lattice_dense")
