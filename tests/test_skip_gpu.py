"""GPU parity of the reduction approximation of the stencil loops (NEXT-3;
PAPER.md §3.3.3, applied to Convolution Separable's two loops,
L1920-1996) against the oracle, and of the extended tuner's decisions.

Tolerance as in test_parity_gpu (reading S18): per output
|gpu - oracle| <= 1e-5 * (oracle skip stencil of |w| on |X|)."""
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


def check(P, O, x, w, sy, sx, xd=None):
    g = P.stencil_skip_xy(dev(x) if xd is None else xd, mkf(P, w), sy, sx).cpu().numpy()
    o = O.stencil_skip_xy(x, w, sy, sx)
    bound = RTOL * O.stencil_skip_xy(np.abs(x), absw(w), sy, sx) + 1e-30
    err = np.abs(g - o)
    assert np.all(err <= bound), (sy, sx, float((err / bound).max()), P.last_kernel())
    return P.last_kernel()


SEP17 = F.separable(17, seed_y=17, seed_x=71)  # the paper's ConvSep: two 1x17 loops (L1650, L1920-1922)
FILTERS = [("gauss3", F.gaussian(3)), ("mean5", F.mean(5)), ("conv9", F.conv(9)), ("signed5", F.conv_signed(5)),
           ("sep7", F.separable(7)), ("sep17", SEP17), ("rect3x7", F.conv(7, seed=11, ky=3))]


@pytest.mark.parametrize("name,w", FILTERS, ids=[f[0] for f in FILTERS])
def test_all_rates(P, O, name, w):
    x = W.frames(2, 77, 300, 5)
    k = (w[0].size if isinstance(w, tuple) else w.shape[0])
    for sy, sx in [(1, 1), (2, 1), (1, 2), (2, 2), (3, 3), (k, 1), (1, k + 3), (4, 2)]:
        check(P, O, x, w, sy, sx)


def test_convsep_fast_path(P, O):
    """Every candidate of the ConvSep tuner runs in a radius-8 tile instance."""
    x = W.frames(1, 190, 700, 2)
    f = mkf(P, SEP17)
    for scheme, rate in P.tune_candidates_ex(f, 3):
        g = P.stencil_approx(dev(x), f, scheme, rate).cpu().numpy()
        o = O.stencil_scheme(x, SEP17, scheme, rate)
        bound = RTOL * O.stencil_scheme(np.abs(x), absw(SEP17), scheme, rate) + 1e-30
        assert np.all(np.abs(g - o) <= bound), (scheme, rate)
        assert P.last_kernel().startswith(("sep8_", "sep_map")), (scheme, rate, P.last_kernel())


def test_schemes_map_to_rates(P):
    x = dev(W.frames(1, 64, 96, 1))
    f = P.Filter(F.mean(5))
    assert torch.equal(P.stencil_approx(x, f, "skip_row", 2), P.stencil_skip_xy(x, f, 2, 1))
    assert torch.equal(P.stencil_approx(x, f, "skip_col", 3), P.stencil_skip_xy(x, f, 1, 3))
    assert torch.equal(P.stencil_approx(x, f, "skip_both", 2), P.stencil_skip_xy(x, f, 2, 2))
    assert torch.equal(P.stencil_skip_xy(x, f, 1, 1), P.stencil_exact(x, f))


def test_stripes_with_halos(P, O):
    """Skip plans keep the full halo: a stripe with halos computes the rows of the whole image."""
    w = SEP17
    x = W.frames(1, 120, 256, 9)[0]
    f = mkf(P, w)
    full = P.stencil_skip_xy(dev(x), f, 3, 2)
    r0, r1 = 40, 80
    stripe = dev(x[r0 - 8:r1 + 8])
    got = P.stencil_skip_xy(stripe, f, 3, 2, halo_top=8, halo_bottom=8)
    assert torch.equal(got, full[r0:r1])


TUNE = [("gauss3", F.gaussian(3), "mre", (8, 192, 256)), ("mean5", F.mean(5), "mre", (8, 192, 256)),
        ("conv9", F.conv(9), "l2", (4, 192, 256)), ("sep7", F.separable(7), "l2", (4, 216, 384)),
        ("sep17", SEP17, "l2", (4, 256, 256))]


@pytest.mark.parametrize("name,w,metric,shape", TUNE, ids=[t[0] for t in TUNE])
@pytest.mark.parametrize("flags", [2, 3])
def test_tuner_ex_bit_identical(P, O, name, w, metric, shape, flags):
    x = W.frames(*shape, seed0=0)
    f = mkf(P, w)
    xd = dev(x)
    parts = P.tune_partials_ex(xd, f, metric, flags)
    ref = O.tune_ex(x, w, 2.0, metric, flags=flags, all_qualities=True)["qualities"]
    qs = [P.quality_from_partials(parts[3 * k:3 * k + 3], metric) for k in range(len(ref))]
    np.testing.assert_allclose(qs, ref, rtol=0, atol=1e-7)
    for toq in (0.80, 0.90, 0.95, 0.99):
        got = P.tune_ex(xd, f, toq, metric, flags)
        o = O.tune_ex(x, w, toq, metric, flags=flags)
        assert got[:2] == (o["scheme"], o["reach"]), (toq, got, o, min(abs(q - toq) for q in ref))
        assert P.tune_decide_ex(f, parts, toq, metric, flags) == got


def test_convsep_2048_full_frame(P, O):
    """The paper's ConvSep workload size (2048^2, L1650) at skip 2 on both loops."""
    x = W.image(2048, 2048, 3)[None]
    assert check(P, O, x, SEP17, 2, 2).startswith("sep8_")
