"""Seeded fuzz of the stencil paths on random shapes, filters and reaches:
dense plans through the tile / map kernels (aligned copy) and through the
fallback kernel (a copy shifted by one float, not TMA-describable) must agree
bit for bit (same per-pixel tap order), and both must meet the S18 bound
against the oracle; separable plans against the oracle (the fallback expands
them to their outer product, so its rounding differs)."""
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


def _misaligned_copy(x):
    buf = torch.zeros(x.numel() + 1, device="cuda")
    v = buf[1:].view(x.shape)
    v.copy_(x)
    return v


DENSE = [F.gaussian(3), F.mean(5), F.conv(7, seed=5), F.conv(9), F.conv_signed(5), F.conv(7, seed=9, ky=3),
         F.conv(3, seed=10, ky=9)]
SEPS = [F.separable(3, 1, 2), F.separable(7), F.separable(9, 3, 4), F.separable(17, 5, 6)]


@pytest.mark.parametrize("trial", range(24))
def test_fuzz_dense_tile_vs_fallback_vs_oracle(P, O, trial):
    rng = np.random.default_rng(1000 + trial)
    n, h, w = int(rng.integers(1, 4)), int(rng.integers(1, 600)), int(rng.integers(1, 700))
    wt = DENSE[int(rng.integers(0, len(DENSE)))]
    ry, rx = wt.shape[0] // 2, wt.shape[1] // 2
    dy, dx = int(rng.integers(0, ry + 2)), int(rng.integers(0, rx + 2))
    x = W.images.random_integers((n, h, w), seed=trial, lo=16, hi=235)
    f = P.Filter(wt)
    xd = torch.from_numpy(x).cuda()
    a = P.stencil_approx_xy(xd, f, dy, dx)
    ka = P.last_kernel()
    mis = _misaligned_copy(xd)
    out = torch.zeros(n * h * w + 1, device="cuda")[1:].view(n, h, w)
    b = P.stencil_approx_xy(mis, f, dy, dx, out=out)
    assert torch.equal(a, b), (trial, (n, h, w), wt.shape, dy, dx, ka, P.last_kernel())
    o = O.stencil_approx_xy(x, wt, dy, dx)
    bound = RTOL * O.stencil_approx_xy(np.abs(x), np.abs(wt), dy, dx) + 1e-30
    assert np.all(np.abs(a.cpu().numpy() - o) <= bound), (trial, ka)


@pytest.mark.parametrize("trial", range(12))
def test_fuzz_separable_vs_oracle(P, O, trial):
    rng = np.random.default_rng(2000 + trial)
    n, h, w = int(rng.integers(1, 3)), int(rng.integers(1, 500)), int(rng.integers(4, 600))
    wy, wx = SEPS[int(rng.integers(0, len(SEPS)))]
    r = wy.size // 2
    dy, dx = int(rng.integers(0, r + 2)), int(rng.integers(0, r + 2))
    x = W.images.random_integers((n, h, w), seed=50 + trial, lo=16, hi=235)
    f = P.Filter(wy=wy, wx=wx)
    g = P.stencil_approx_xy(torch.from_numpy(x).cuda(), f, dy, dx).cpu().numpy()
    o = O.stencil_sep(x, wy, wx, dy, dx)
    bound = RTOL * O.stencil_sep(np.abs(x), np.abs(wy), np.abs(wx), dy, dx) + 1e-30
    assert np.all(np.abs(g - o) <= bound), (trial, (n, h, w), wy.size, dy, dx, P.last_kernel())
